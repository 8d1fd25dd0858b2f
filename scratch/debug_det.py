import sys, os
sys.path.insert(0, '.')
import numpy as np, torch
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
w = gen.CONFIGS[os.environ.get("CFG", "C5")]
st = runner.Stack(w, "cuda")
outs = []
for r in range(4):
    st.forward(inference=(r % 2 == 1)); torch.cuda.synchronize()
    outs.append(st.H[w.layers].clone())
for r in range(1, 4):
    d = (outs[r] != outs[0])
    nbad = int(d.sum())
    rows = torch.nonzero(d.any(1)).flatten()
    print("run", r, "differs in", nbad, "entries,", rows.numel(), "rows", rows[:10].tolist(), flush=True)
# check the projection separately: saved P across runs
sv = st.saved[0]
st.forward(); torch.cuda.synchronize(); p1 = sv.clone()
st.forward(); torch.cuda.synchronize(); p2 = sv.clone()
nP = w.n * w.k
P1 = p1[:nP*4].view(torch.float32); P2 = p2[:nP*4].view(torch.float32)
print("saved P differs:", int((P1 != P2).sum()), flush=True)
