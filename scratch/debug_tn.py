import sys, os
sys.path.insert(0, '.')
import numpy as np, torch
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M, K1, N = 32, 128, 128
A = torch.zeros((M, K1)); 
for r in range(M): A[r, r] = 1.0
B = torch.arange(M * N, dtype=torch.float32).reshape(M, N) / 1000.0 + 1.0
C = torch.full((K1, N), float('nan'), device='cuda')
agnn.debug_gemm_tn(A.cuda(), B.cuda(), C)
torch.cuda.synchronize()
c = C.cpu().numpy(); ref = (A.T @ B).numpy()
print("desc", os.environ.get("AGNN_TN_DESC"), "max err", np.abs(c - ref).max())
nz = np.argwhere(np.abs(c) > 1e-6)
print("nonzero rows:", sorted(set(nz[:, 0].tolist()))[:40])
for k1 in [0, 1, 2, 7, 8, 31]:
    row = c[k1]
    # identify which B row/cols it matches
    m = [(r, int(np.argmin(np.abs(B.numpy()[r] - row[0])))) for r in range(M) if np.any(np.isclose(B.numpy()[r], row[0]))]
    print(k1, row[:4], "ref", ref[k1, :4], "match(row,col) of c[k1,0]:", m[:3])
