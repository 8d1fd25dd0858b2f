import os, sys, dataclasses
sys.path.insert(0, '.'); sys.path.insert(0, 'oracle'); sys.path.insert(0, 'tests')
import numpy as np, torch
import parity_utils as pu
from paper_conf_sc_bestarglzcgssci23_b200 import gen
def W(model, graph, scale, ef, k, heads=1, layers=1, act="relu", n=None, samples=None, **kw):
    n = n or (1 << scale)
    return gen.Workload(f"{model}-{graph}{scale}-k{k}h{heads}L{layers}", model, graph, scale, n,
                        samples if samples is not None else ef * n, k, heads, layers, act=act, **kw)
cases = [W("gat","kron",15,8,128,heads=4), W("gat","kron",15,8,128,heads=1), W("gat","kron",15,8,64,heads=1,act="none"),
         W("gat","kron",12,8,128,heads=4), W("gat","er",0,0,128,heads=4,n=4000,samples=30000), gen.CONFIGS["C2"]]
for w in cases:
    src, dst, rp, ci = pu.host_graph(w)
    H, Ws, As, R = w.host_inputs()
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    for chunk in ("2048", "100000000", "64"):
        os.environ["AGNN_CHUNK_EDGES"] = chunk
        g = pu.device_graph(w, src, dst)
        st = pu.gpu_step(w, graph=g)
        try:
            errs = pu.compare(w, st, ref, tol=1e9)
        except AssertionError as e:
            errs = str(e)
        print(w.name, "chunk", chunk, "maxdeg", np.diff(rp).max(), {k: f"{v:.1e}" for k, v in errs.items()}, flush=True)
