"""Inference-forward time at C5 (fp32): the register-gather k'=128 kernel vs the TMA
gather4 variant (AGNN_GATHER=tma), via the library's live per-kernel profile."""
import os, sys, json, torch
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
from paper_conf_sc_bestarglzcgssci23_b200 import agnn, gen, runner
w = gen.CONFIGS["C5"]
st = runner.Stack(w, "cuda")
for _ in range(2):
    st.forward(inference=True)
torch.cuda.synchronize()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
ev[0].record()
for _ in range(5):
    st.forward(inference=True)
ev[1].record()
torch.cuda.synchronize()
print(os.environ.get("AGNN_GATHER", "reg"), "inference forward ms:", round(ev[0].elapsed_time(ev[1]) / 5, 2))
