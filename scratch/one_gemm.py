import sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import agnn
M = 1 << 22
A = torch.rand((M, 128), device="cuda") - 0.5
W = torch.rand((128, 128), device="cuda") - 0.5
C = torch.empty((M, 128), device="cuda")
B = torch.rand((M, 128), device="cuda") - 0.5
Ct = torch.empty((128, 128), device="cuda")
agnn.debug_gemm(A, W, C); agnn.debug_gemm_tn(A, B, Ct)
torch.cuda.synchronize()
