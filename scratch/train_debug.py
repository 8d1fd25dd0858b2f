import dataclasses, sys
import numpy as np, torch
sys.path.insert(0, "tests"); sys.path.insert(0, "oracle")
import parity_utils as pu
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
model, heads = sys.argv[1], int(sys.argv[2])
w = dataclasses.replace(gen.Workload(f"train-{model}", model, "kron", 12, 1 << 12, 8 << 12, 32, heads, 2,
                                     act="elu"), train=True, lr=0.05)
src, dst, rp, ci = pu.host_graph(w)
g = pu.device_graph(w, src, dst)
st = runner.Stack(w, "cuda", graph=g)
H, Ws, As, R = w.host_inputs()
Ws = [x.astype(np.float64) for x in Ws]; As = [None if x is None else x.astype(np.float64) for x in As]
for it in range(4):
    # compare GPU weights before the step with the oracle's
    print("it", it, "W err", [pu.rel(st.W[l].cpu().numpy(), Ws[l]) for l in range(2)],
          "a err", [pu.rel(st.a[l].cpu().numpy(), As[l]) for l in range(2)] if As[0] is not None else "")
    print("  |a|max", [float(np.abs(As[l]).max()) for l in range(2)] if As[0] is not None else "",
          "|W|max", [float(np.abs(Ws[l]).max()) for l in range(2)])
    st.forward(); st.backward()
    torch.cuda.synchronize()
    ref = pu.oracle_step(w, rp, ci, H, [x.astype(np.float32).astype(np.float64) for x in Ws] if False else Ws, As, R)
    errs = {}
    for l in range(1, 3): errs[f"H{l}"] = pu.rel(st.H[l].cpu().numpy(), ref["H"][l])
    for l in range(3): errs[f"dH{l}"] = pu.rel(st.dH[l].cpu().numpy(), ref["dH"][l])
    for l in range(2):
        errs[f"dW{l}"] = pu.rel(st.dW[l].cpu().numpy(), ref["dW"][l])
        if As[0] is not None: errs[f"da{l}"] = pu.rel(st.da[l].cpu().numpy(), ref["da"][l])
    print("  ", {k: f"{v:.2e}" for k, v in errs.items()})
    f = ref["fwd"][0]
    if "alpha" in f:
        print("   alpha min/max", float(f["alpha"].min()), float(f["alpha"].max()))
    st.sgd(); torch.cuda.synchronize()
    for l in range(2):
        Ws[l] = Ws[l] - w.lr * ref["dW"][l]
        if As[l] is not None: As[l] = As[l] - w.lr * ref["da"][l]
