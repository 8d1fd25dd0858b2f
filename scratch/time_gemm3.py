"""k = 256 projection (C4 shape): C[M x N] = A[M x 256] B^T, M = 2^22."""
import os, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M = 1 << 22
A = torch.rand((M, 256), device="cuda") - 0.5
out = []
for N in (128, 256):
    W = torch.rand((N, 256), device="cuda") - 0.5
    C = torch.empty((M, N), device="cuda")
    for _ in range(2): agnn.debug_gemm(A, W, C)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10): agnn.debug_gemm(A, W, C)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    out.append(f"K=256 N={N}: {ms:.3f} ms ({M*(256+N)*4/ms/1e6:.0f} GB/s)")
print(os.environ.get("AGNN_LIB", "tree"), " | ".join(out))
