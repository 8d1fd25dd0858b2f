"""Training vs inference forward H_out: which rows differ (factored GAT forward)."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np, torch
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
for prec in ("fp32", "bf16"):
    for act in ("elu", "relu"):
        w = gen.Workload(f"dbg-{prec}", "gat", "kron", 13, 1 << 13, 8 << 13, 128, 4, 1, act=act, prec=prec)
        st = runner.Stack(w, "cuda")
        st.step()
        a = st.H[1].clone()
        st.H[1].zero_()
        st.forward(inference=True)
        torch.cuda.synchronize()
        d = (a != st.H[1]).any(dim=1).cpu().numpy()
        rp = st.row_ptr.cpu().numpy()
        deg = np.diff(rp)
        bad = np.nonzero(d)[0]
        print(prec, act, "rows differing:", len(bad), "degrees:", np.unique(deg[bad])[:20],
              "max abs diff", float((a - st.H[1]).abs().max()))
