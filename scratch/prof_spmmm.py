"""One forward of AGNN k=128 on ER 2^20 with spmmm 0 then 1 (for ncu)."""
import sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
n = 1 << 20
w = gen.Workload("agnn-er", "agnn", "er", 0, n, 16 * n, 128, 1, 1, act="relu")
for sp in (0, 1):
    st = runner.Stack(w, "cuda", plan_options={"spmmm": sp})
    st.forward(); st.forward()
    torch.cuda.synchronize()
    del st
