import os, sys, dataclasses
sys.path.insert(0, '.'); sys.path.insert(0, 'oracle'); sys.path.insert(0, 'tests')
import numpy as np, torch
import parity_utils as pu
from paper_conf_sc_bestarglzcgssci23_b200 import gen
mode = sys.argv[1]
for w in [dataclasses.replace(gen.CONFIGS["C2"], act="elu"), dataclasses.replace(gen.CONFIGS["C2"], act="elu", layers=1),
          dataclasses.replace(gen.CONFIGS["C2"], act="none", layers=1, slope=1.0)]:
    src, dst, rp, ci = pu.host_graph(w)
    H, Ws, As, R = w.host_inputs()
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    g = pu.device_graph(w, src, dst)
    st = pu.gpu_step(w, graph=g)
    errs = pu.compare(w, st, ref, tol=1e9)
    # near-kink edges in the oracle
    f = ref["fwd"][-1]
    pre = f["s"][np.repeat(np.arange(w.n), np.diff(rp))] + f["t"][ci]
    print(mode, w.name, w.layers, w.act, w.slope, {k: f"{v:.1e}" for k, v in errs.items()}, "min|pre|", np.abs(pre).min(), flush=True)
