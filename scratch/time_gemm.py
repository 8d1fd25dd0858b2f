"""Time the library's GEMMs at the C5 shapes (M = 2^24, K = N = 128) with CUDA events.
AGNN_LIB selects the libagnn.so under test."""
import os, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M = 1 << 24
A = torch.rand((M, 128), device="cuda") - 0.5
B = torch.rand((M, 128), device="cuda") - 0.5
W = torch.rand((144, 128), device="cuda") - 0.5
C = torch.empty((128, 128), device="cuda")
C2 = torch.empty((M, 144), device="cuda")
def t(f, n=10):
    for _ in range(2): f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(n): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n
tn = t(lambda: agnn.debug_gemm_tn(A, B, C))
tc = t(lambda: agnn.debug_gemm(A, W, C2))
print(f"{os.environ.get('AGNN_LIB','tree')}: gemm_tn {tn:.3f} ms ({2*M*128*4/tn/1e6:.0f} GB/s)  "
      f"gemm_tc N=144 {tc:.3f} ms ({M*(128+144)*4/tc/1e6:.0f} GB/s)")
