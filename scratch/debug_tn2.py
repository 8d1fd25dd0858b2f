import sys, os
sys.path.insert(0, '.')
import numpy as np, torch
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M, K1, N = 32, 128, 128
A = torch.arange(M * K1, dtype=torch.float32).reshape(M, K1) + 1.0
B = torch.ones((M, N))
C = torch.full((K1, N), float('nan'), device='cuda')
agnn.debug_gemm_tn(A.cuda(), B.cuda(), C)
torch.cuda.synchronize()
c = C.cpu().numpy().ravel()
print("desc", os.environ.get("AGNN_TN_DESC"), "first values", c[:40])
print("A row0", A[0, :8].numpy(), "A row1", A[1, :8].numpy())
ref = (A.T @ B).numpy()
print("ref", ref[:2, :4])
