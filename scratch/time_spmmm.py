"""A/B of the AGNN/VA k=128 forward: SpMM kernel + tcgen05 GEMM vs the fused SpMMM
kernel, on several synthetic graphs (forward only, CUDA events, median of 10)."""
import sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner

def W(model, graph, scale, ef, n=None):
    n = n or (1 << scale)
    return gen.Workload(f"{model}-{graph}{scale}", model, graph, scale, n, ef * n, 128, 1, 1, act="relu")

cases = [W("agnn", "er", 0, 16, n=1 << 20), W("agnn", "rmat", 20, 16), W("agnn", "kron", 20, 16),
         W("va", "kron", 20, 16), W("agnn", "kron", 22, 32)]
for w in cases:
    res = {}
    for sp in (0, 1):
        st = runner.Stack(w, "cuda", plan_options={"spmmm": sp})
        for inf in (False, True):
            for _ in range(3):
                st.forward(inference=inf)
            ts = []
            for _ in range(10):
                a, b = torch.cuda.Event(True), torch.cuda.Event(True)
                a.record(st.stream); st.forward(inference=inf); b.record(st.stream)
                torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
            res[(sp, inf)] = sorted(ts)[5]
        info = st.plan.info()
        del st
        torch.cuda.empty_cache()
    print(f"{w.name}: m={info['nnz']} heavy={info['heavy_rows']} chunks={info['heavy_chunks']} "
          f"train split {res[(0, False)]:.3f} fused {res[(1, False)]:.3f} | "
          f"infer split {res[(0, True)]:.3f} fused {res[(1, True)]:.3f} ms", flush=True)
