"""Rows each rank receives per exchange with the needed-rows all-gather (comm.cu) vs
the full all-gather, for the 1D row-block partition at P = 2/4/8 (reading A20)."""
import json, sys, torch
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import agnn, gen, runner
out = {}
for cfg in sys.argv[1:] or ["C3", "C4", "C5"]:
    w = gen.CONFIGS[cfg]
    g = runner.build_graph(w, torch.device("cuda"))
    rp = g.row_ptr.cpu().numpy()
    res = {}
    for P in (2, 4, 8):
        b = agnn.partition(rp, P, 4)
        recv = []
        for r in range(P):
            e0, e1 = int(rp[b[r]]), int(rp[b[r + 1]])
            cols = torch.unique(g.col_idx[e0:e1])
            recv.append(int(((cols < int(b[r])) | (cols >= int(b[r + 1]))).sum()))
        full = [int(w.n - (b[r + 1] - b[r])) for r in range(P)]
        res[P] = {"recv_max": max(recv), "recv_mean": sum(recv) / P, "full_max": max(full),
                  "ratio_max": max(recv) / max(full), "rows_max": int(max(b[1:] - b[:-1])),
                  "edges_max": int(max(rp[b[1:]] - rp[b[:-1]]))}
    out[cfg] = {"n": w.n, "m": g.nnz, "P": res}
    print(cfg, json.dumps(out[cfg]), flush=True)
    del g
    torch.cuda.empty_cache()
json.dump(out, open("gpurun_out/exchange_volume.json", "w"), indent=1)
