import sys, os
sys.path.insert(0, '.')
import numpy as np, torch
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner, agnn
import dataclasses
w = dataclasses.replace(gen.CONFIGS[os.environ.get("CFG", "C5")], act="none")
st = runner.Stack(w, "cuda")
st.forward(); st.backward(); torch.cuda.synchronize()
g = torch.Generator(device="cuda").manual_seed(11)
V = torch.randn(st.W[0].shape, device="cuda", generator=g) * 1e-2
v = torch.randn(st.a[0].shape, device="cuda", generator=g) * 1e-2
predW = float((st.dW[0].double() * V.double()).sum()); preda = float((st.da[0].double() * v.double()).sum())
np.save(f"gpurun_out/dW_{os.environ.get('AGNN_GEMM','tc')}.npy", st.dW[0].cpu().numpy())
print(os.environ.get("AGNN_GEMM","tc"), "predW", predW, "preda", preda, flush=True)
W0, a0 = st.W[0].clone(), st.a[0].clone(); R = st.dH[w.layers]
def loss(eW, ea):
    st.W[0].copy_(W0 + eW * V); st.a[0].copy_(a0 + ea * v); st.forward(inference=True)
    return float((st.H[w.layers].double() * R.double()).sum())
for eps in [0.2, 0.1, 0.05, 0.02]:
    fdW = (loss(eps, 0) - loss(-eps, 0)) / (2 * eps)
    fda = (loss(0, eps) - loss(0, -eps)) / (2 * eps)
    print("eps", eps, "fdW", fdW, "fda", fda, flush=True)
