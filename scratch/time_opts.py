"""C5 step time under plan work-decomposition options (short_edges, chunk_edges):
python scratch/time_opts.py  (CUDA events, median of 5 steps after 3 warm-ups)."""
import sys, json, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner

w = gen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C5"]
g = runner.build_graph(w, torch.device("cuda"))
variants = [{}, {"short_edges": 16}, {"short_edges": 24}, {"chunk_edges": 1024},
            {"chunk_edges": 4096}, {}]
for opts in variants:
    st = runner.Stack(w, "cuda", graph=g, plan_options=opts or None)
    for _ in range(3):
        st.step()
    ts = []
    for _ in range(5):
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record(st.stream); st.step(); b.record(st.stream)
        torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    print(json.dumps({"opts": opts, "ms": sorted(ts)[2], "all": [round(t, 2) for t in ts]}), flush=True)
    del st
    torch.cuda.empty_cache()
