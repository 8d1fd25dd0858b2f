"""Full-size parity of the AGNN / VA path at the bench configurations C3 (AGNN,
R-MAT 2^20, k = 128, 3 layers) and C4 (VA, Kronecker 2^22, k = 256), and of C5 in
the BF16 storage mode (the bench line's `bf16_storage`, reading B1, bar 1e-2), in
the launch configuration bench.py times, on outputs the oracle computes from exact
local sub-problems (the argument of test_gpu_fullsize.py):

  * forward: row i of layer 0 depends only on H of N(i) u {i}, so the oracle runs
    on a sub-CSR holding the sampled rows' complete neighbour lists (uniform light
    rows, the maximum-degree row and rows of several heavy-row chunks);
  * backward of layer 0, EXACT at full size: with the upstream gradient R
    supported on a row set S, G and M = G W^T vanish outside S, so dH (PAPER.md
    Eq. 11 for VA; the cosine-softmax backward of reading A8 for AGNN) is
    non-zero only on S u N(S) and depends only on the complete rows of S and the
    features of S u N(S), and dW = X^T G only on the rows of S: the oracle computes
    dH of the WHOLE graph and dW from that 1-hop sub-problem, and every dH row
    outside S u N(S) must be exactly 0.
"""
from __future__ import annotations

import dataclasses

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]

import oracle  # noqa: E402
import parity_utils as pu  # noqa: E402
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner  # noqa: E402
from test_gpu_fullsize import _hub_rows, _neighbours, _subproblem  # noqa: E402


@pytest.fixture(scope="module", params=["C3", "C4", "C5-bf16"])
def stack(request):
    if request.param == "C5-bf16":
        w = dataclasses.replace(gen.CONFIGS["C5"], prec="bf16")
    else:
        w = gen.CONFIGS[request.param]
    st = runner.Stack(w, "cuda")
    st.forward()
    torch.cuda.synchronize()
    rp = st.row_ptr.cpu().numpy()
    yield w, st, rp
    del st
    torch.cuda.empty_cache()


def _layer0_inputs(w, sources):
    H = gen.fill_rows(w.seed, gen.STREAM_H, np.asarray(sources, np.int64), w.k, 1.0)
    wshape, ashape = w.weight_shapes(0)
    bound = gen.glorot_bound(w.k, w.k)
    W0 = gen.fill(w.seed, gen.STREAM_W(0), wshape, bound)
    a0 = gen.fill(w.seed, gen.STREAM_A(0), ashape, bound) if ashape else None
    return H, W0, a0


def _oracle_forward(w, srp, sci, H, W0, a0):
    f, _ = oracle.layer(w.model, srp, sci, np.asarray(H, np.float64), W0, a0, w.heads, act=w.act,
                        slope=w.slope, beta=w.beta, eps=w.eps, agg=w.agg, bf16=w.prec == "bf16")
    return f


def _bars(w):
    """FP32: 1e-5 normwise + per-row bounds; BF16 storage: 1e-2 and forward rows only
    (pu.rowwise_keys: one-ulp bf16 decisions move single backward rows)."""
    if w.prec == "bf16":
        return dict(tol=pu.TOL_BF16, row_tol=pu.BF16_ROW_TOL), False
    return dict(tol=pu.TOL_FP32), True


def test_forward_sampled_rows(stack):
    w, st, rp = stack
    rng = np.random.default_rng(7)
    deg = np.diff(rp)
    chunk = st.plan.info()["chunk"]
    hubs = _hub_rows(rp, chunk, rng)
    assert deg[hubs[0]] > 20 * chunk
    light = rng.choice(np.nonzero(deg <= chunk)[0], 128, replace=False)
    rows = np.unique(np.concatenate([light, hubs])).astype(np.int64)
    nbs = _neighbours(st, rp, rows)
    sources = np.union1d(np.unique(np.concatenate(nbs)), rows)
    srp, sci = _subproblem(rp, nbs, rows, sources)
    H, W0, a0 = _layer0_inputs(w, sources)
    f = _oracle_forward(w, srp, sci, H, W0, a0)
    pos = np.searchsorted(sources, rows)
    got = st.H[1][torch.from_numpy(rows).cuda()].cpu().numpy()
    hub = np.isin(rows, hubs)
    bars, _ = _bars(w)
    pu.compare_arrays({"Hout": (got, f["Hout"][pos]), "Hout_hubs": (got[hub], f["Hout"][pos][hub])},
                      rowwise=["Hout", "Hout_hubs"], **bars)


def test_backward_exact_on_row_support(stack):
    w, st, rp = stack
    rng = np.random.default_rng(8)
    deg = np.diff(rp)
    chunk = st.plan.info()["chunk"]
    hubs = [r for r in _hub_rows(rp, chunk, rng)[1:] if deg[r] <= 4 * chunk][:2]
    cand = rng.choice(np.nonzero((deg >= 2) & (deg <= 32))[0], 20000, replace=False)
    nxt, plain = [], []
    for j in cand:
        nb = st.col_idx[rp[j]:rp[j + 1]].cpu().numpy()
        if len(nxt) < 16 and deg[nb].max() > chunk:
            nxt.append(int(j))
        elif len(plain) < 16 and deg[nb].max() <= chunk:
            plain.append(int(j))
        if len(nxt) == 16 and len(plain) == 16:
            break
    S = np.unique(np.array(hubs + nxt + plain, np.int64))
    nbs = _neighbours(st, rp, S)
    sources = np.union1d(np.unique(np.concatenate(nbs)), S)  # S u N(S)
    srp, sci = _subproblem(rp, nbs, S, sources)
    H, W0, a0 = _layer0_inputs(w, sources)
    f = _oracle_forward(w, srp, sci, H, W0, a0)
    posS = np.searchsorted(sources, S)
    # ReLU kink (reading A6'): zero R where the oracle's Z is within 1e-5 rms of 0
    RS = gen.fill_rows(w.seed, gen.STREAM_R, S, w.k, 1.0).astype(np.float64)
    ZS = f["Z"][posS]
    RS[np.abs(ZS) < 1e-5 * np.sqrt(np.mean(ZS ** 2))] = 0.0
    R = np.zeros((len(sources), w.k))
    R[posS] = RS
    Hs = np.asarray(H, np.float64)
    bf = w.prec == "bf16"
    if w.model == "agnn":
        b = oracle.agnn_backward(srp, sci, Hs, W0, f, R, w.beta, w.eps, w.act, bf16=bf)
    elif w.model == "gat":
        b = oracle.gat_backward(srp, sci, Hs, W0, a0, w.heads, f, R, w.slope, w.act, bf16=bf)
    else:
        b = oracle.va_backward(srp, sci, Hs, W0, f, R, w.act, bf16=bf)
    # the GPU backward of layer 0 (forward state of the bench's stack) with that R
    dH1 = torch.zeros_like(st.dH[1])
    dH1[torch.from_numpy(S).cuda()] = torch.from_numpy(RS.astype(np.float32)).cuda()
    st.model.backward(0, st.W[0], st.a[0], st.H[0], st.saved[0], dH1, st.dH[0], st.dW[0],
                      st.da[0], st.ws, st.stream)
    torch.cuda.synchronize()
    dH = st.dH[0]
    src_t = torch.from_numpy(sources).cuda()
    got_dH = dH[src_t].cpu().numpy()
    outside = torch.ones(w.n, dtype=torch.bool, device="cuda")
    outside[src_t] = False
    nonzero_outside = int((dH[outside] != 0).any(dim=1).sum())
    pairs = {"dH_support": (got_dH, b["dH"]), "dH_S": (got_dH[posS], b["dH"][posS]),
             "dW": (st.dW[0].cpu().numpy(), b["dW"])}
    if w.model == "gat":
        pairs["da"] = (st.da[0].cpu().numpy(), b["da"])
    bars, rowwise = _bars(w)
    pu.compare_arrays(pairs, rowwise=["dH_support", "dH_S", "dW"] if rowwise else [], **bars)
    assert nonzero_outside == 0, nonzero_outside
