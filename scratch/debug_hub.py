import sys, os, time
sys.path.insert(0, '.'); sys.path.insert(0, 'oracle'); sys.path.insert(0, 'tests')
import numpy as np, torch
import oracle
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
import test_gpu_fullsize as T
w = gen.CONFIGS[os.environ.get("CFG", "C5")]
st = runner.Stack(w, "cuda"); st.forward(); torch.cuda.synchronize()
rp = st.row_ptr.cpu().numpy(); deg = np.diff(rp)
order = np.argsort(-deg)
print("top degrees", deg[order[:5]], "chunks", st.plan.info(), flush=True)
for rows in [order[:2], order[100:102], order[3000:3002]]:
    rows = np.sort(rows)
    nb = np.unique(np.concatenate([st.col_idx[rp[r]:rp[r + 1]].cpu().numpy() for r in rows]))
    sources = np.union1d(nb, rows)
    t0 = time.time()
    srp, sci = T._subproblem(rp, st.col_idx, rows, sources)
    H = gen.fill(w.seed, gen.STREAM_H, (w.n, w.k)) if len(sources) > 200000 else T._host_rows(w.seed, gen.STREAM_H, sources, w.k)
    if H.shape[0] == w.n: H = H[sources]
    Wt = gen.fill(w.seed, gen.STREAM_W(0), (w.k, w.k), gen.glorot_bound(w.k, w.k))
    at = gen.fill(w.seed, gen.STREAM_A(0), (w.heads, 2 * (w.k // w.heads)), gen.glorot_bound(w.k, w.k))
    f = oracle.gat_forward(srp, sci, H, Wt, at, w.heads, w.slope, w.act)
    pos = np.searchsorted(sources, rows)
    ref = f["Hout"][pos]
    got = st.H[1][torch.from_numpy(rows).cuda()].cpu().numpy().astype(np.float64)
    print("rows deg", deg[rows], "fwd rel err", np.linalg.norm(got - ref) / np.linalg.norm(ref), "t", time.time()-t0, flush=True)
# directional derivative check with several eps
st.forward(); st.backward(); torch.cuda.synchronize()
g = torch.Generator(device="cuda").manual_seed(11)
V = torch.randn(st.W[0].shape, device="cuda", generator=g) * 1e-2
v = torch.randn(st.a[0].shape, device="cuda", generator=g) * 1e-2
pW = float((st.dW[0].double() * V.double()).sum()); pa = float((st.da[0].double() * v.double()).sum())
W0, a0 = st.W[0].clone(), st.a[0].clone(); R = st.dH[w.layers]
def loss(eW, ea):
    st.W[0].copy_(W0 + eW * V); st.a[0].copy_(a0 + ea * v); st.forward(inference=True)
    return float((st.H[1].double() * R.double()).sum())
L0 = loss(0, 0)
for eps in [0.2, 0.05, 0.01]:
    fdW = (loss(eps, 0) - loss(-eps, 0)) / (2 * eps)
    fda = (loss(0, eps) - loss(0, -eps)) / (2 * eps)
    print("eps", eps, "L0", L0, "fdW", fdW, "predW", pW, "fda", fda, "preda", pa, flush=True)
print("|dW|", float(st.dW[0].norm()), "|da|", float(st.da[0].norm()))
