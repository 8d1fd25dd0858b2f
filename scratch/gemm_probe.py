"""Accuracy and timing probe of the projection GEMMs (debug_gemm / debug_gemm_tn)."""
import sys
import numpy as np
import torch
from paper_conf_sc_bestarglzcgssci23_b200 import agnn

def acc(M, K, N, tn=False):
    g = torch.Generator().manual_seed(1)
    if tn:
        A = (torch.rand((M, K), generator=g) * 2 - 1).cuda()
        B = (torch.rand((M, N), generator=g) * 2 - 1).cuda()
        C = torch.empty((K, N), device="cuda")
        agnn.debug_gemm_tn(A, B, C)
        ref = A.double().T @ B.double()
        scale = A.double().abs().T @ B.double().abs()
    else:
        A = (torch.rand((M, K), generator=g) * 2 - 1).cuda()
        B = ((torch.rand((N, K), generator=g) * 2 - 1) * K ** -0.5).cuda()
        C = torch.empty((M, N), device="cuda")
        agnn.debug_gemm(A, B, C)
        ref = A.double() @ B.double().T
        scale = A.double().abs() @ B.double().abs().T
    err = (C.double() - ref)
    print(f"{'TN' if tn else 'NT'} M={M} K={K} N={N}: norm {float(err.norm() / ref.norm()):.3e} "
          f"max/scale {float((err.abs() / scale).max()):.3e}", flush=True)

def timing(M, K, N, tn=False, reps=10):
    A = torch.rand((M, K), device="cuda")
    if tn:
        B = torch.rand((M, N), device="cuda"); C = torch.empty((K, N), device="cuda")
        f = lambda: agnn.debug_gemm_tn(A, B, C)
    else:
        B = torch.rand((N, K), device="cuda"); C = torch.empty((M, N), device="cuda")
        f = lambda: agnn.debug_gemm(A, B, C)
    f(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        f()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    byts = (M * K + (K * N if tn else M * N) + (M * N if tn else 0)) * 4
    print(f"{'TN' if tn else 'NT'} M={M} K={K} N={N}: {ms:.3f} ms  {byts / ms / 1e6:.0f} GB/s", flush=True)

if __name__ == "__main__":
    mode = sys.argv[1] if len(sys.argv) > 1 else "all"
    if mode in ("all", "acc"):
        for M, K, N in [(100003, 128, 128), (100003, 128, 144), (100003, 256, 256), (100003, 256, 128)]:
            acc(M, K, N)
        for M, K, N in [(100003, 128, 128), (100003, 256, 256)]:
            acc(M, K, N, tn=True)
    if mode in ("all", "time"):
        for M, K, N in [(1 << 24, 128, 144), (1 << 24, 128, 128), (1 << 22, 256, 256)]:
            timing(M, K, N)
        for M, K, N in [(1 << 24, 128, 128), (1 << 22, 256, 256)]:
            timing(M, K, N, tn=True)
    if mode == "ncu":
        timing(1 << 22, 256, 256, reps=1)

if __name__ == "__main__" and len(sys.argv) > 1 and sys.argv[1] == "ncu144":
    timing(1 << 24, 128, 144, reps=1)
