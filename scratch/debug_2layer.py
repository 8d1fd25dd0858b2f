"""2-layer GAT k'=128 parity under env variants (factored, bundles, hints)."""
import os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, numpy as np
sys.path[:0] = [%r, %r, %r]
import parity_utils as pu
from paper_conf_sc_bestarglzcgssci23_b200 import gen
w = gen.Workload("g", "gat", "%s", %d, 1 << %d, %d << %d, 128, %d, %d, act="elu")
src, dst, rp, ci = pu.host_graph(w)
g = pu.device_graph(w, src, dst)
st = pu.gpu_step(w, graph=g)
H, Ws, As, R = w.host_inputs()
ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
errs = {}
for l in range(w.layers + 1):
    errs["dH%%d" %% l] = pu.rel(st.dH[l].cpu().numpy(), ref["dH"][l])
for l in range(w.layers):
    errs["dW%%d" %% l] = pu.rel(st.dW[l].cpu().numpy(), ref["dW"][l])
    errs["H%%d" %% (l+1)] = pu.rel(st.H[l+1].cpu().numpy(), ref["H"][l+1])
print({k: float("%%.1e" %% v) for k, v in errs.items()})
'''
cases = [("rmat", 13, 16, 2, 2), ("kron", 13, 8, 4, 2), ("rmat", 13, 16, 2, 1)]
envs = [{}, {"AGNN_GAT_FACTORED": "0"}, {"AGNN_SHORT_BUNDLES": "0"}, {"AGNN_L2_HOT_MB": "0"}, {"AGNN_CHUNK_EDGES": "100000"}]
for (gr, sc, ef, h, L) in cases:
    for e in envs:
        code = CHILD % (ROOT, ROOT + "/tests", ROOT + "/oracle", gr, sc, sc, ef, sc, h, L)
        r = subprocess.run([sys.executable, "-c", code], env=dict(os.environ, **e), capture_output=True, text=True)
        print(gr, sc, "h", h, "L", L, e, r.stdout.strip()[-300:], r.stderr.strip()[-300:] if r.returncode else "")
