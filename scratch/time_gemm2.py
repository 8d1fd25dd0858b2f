"""Projection GEMM time vs N (resident B size -> ring stages): C[M x N] = A[M x 128] B^T."""
import os, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M = 1 << 24
A = torch.rand((M, 128), device="cuda") - 0.5
def t(f, n=10):
    for _ in range(2): f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(n): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
out = []
for N in (64, 128, 144, 160):
    W = torch.rand((N, 128), device="cuda") - 0.5
    C = torch.empty((M, N), device="cuda")
    ms = t(lambda: agnn.debug_gemm(A, W, C))
    out.append(f"N={N}: {ms:.3f} ms ({M*(128+N)*4/ms/1e6:.0f} GB/s)")
    del C
print(os.environ.get("AGNN_LIB", "tree"), " | ".join(out))
