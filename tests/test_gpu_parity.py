"""GPU parity: the CUDA path (through the C ABI) against the FP64 oracle.

Inputs are the seeded synthetic workloads (paper_conf_sc_bestarglzcgssci23_b200.gen)
at sizes the oracle finishes in seconds that still span many tiles, heavy-row
chunks (degree > the plan's chunk size) and ragged tails.  Bars (north_star / SURVEY §8(c)):
  * CSR metadata bit-exact with the oracle's host builder;
  * every float output normwise <= 1e-5 relative (FP32);
  * attention alpha elementwise |a - a_ref| <= 1e-5 a_ref + 1e-9.
"""
from __future__ import annotations

import dataclasses

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]

import oracle  # noqa: E402
import parity_utils as pu  # noqa: E402
from paper_conf_sc_bestarglzcgssci23_b200 import agnn, gen, runner  # noqa: E402


def W(model, graph, scale, ef, k, heads=1, layers=1, act="relu", n=None, samples=None, **kw):
    n = n or (1 << scale)
    return gen.Workload(f"{model}-{graph}{scale}-k{k}h{heads}L{layers}", model, graph, scale, n,
                        samples if samples is not None else ef * n, k, heads, layers, act=act, **kw)


# ------------------------------------------------------------------ CSR metadata
@pytest.mark.parametrize("w", [gen.CONFIGS["C1"], W("gat", "kron", 14, 8, 16),
                               W("gat", "rmat", 13, 16, 16), W("gat", "er", 0, 0, 16, n=3000,
                                                               samples=20000)],
                         ids=lambda w: w.name)
def test_csr_build_bit_exact(w):
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    np.testing.assert_array_equal(g.row_ptr.cpu().numpy(), rp)
    np.testing.assert_array_equal(g.col_idx.cpu().numpy(), ci)


def test_device_generators_match_host():
    w = gen.CONFIGS["C2"]
    s = torch.empty(w.n_samples, dtype=torch.int32, device="cuda")
    d = torch.empty_like(s)
    gen.edges_device(w.kind, w.seed, w.scale, w.n, w.n_samples, s.data_ptr(), d.data_ptr())
    hs, hd = w.host_edges()
    np.testing.assert_array_equal(s.cpu().numpy().view(np.uint32), hs)
    np.testing.assert_array_equal(d.cpu().numpy().view(np.uint32), hd)
    H = torch.empty(1000, 64, device="cuda")
    gen.fill_device(1, gen.STREAM_W(0), H.numel(), gen.glorot_bound(64, 64), H.data_ptr(),
                    offset=0)
    np.testing.assert_array_equal(H.cpu().numpy(), gen.fill(1, gen.STREAM_W(0), (1000, 64),
                                                            gen.glorot_bound(64, 64)))


def test_plan_info_and_heavy_rows():
    w = W("gat", "kron", 16, 8, 64)
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    plan = agnn.Plan(g.row_ptr, g.col_idx, w.n)
    info = plan.info()
    deg = np.diff(rp)
    assert info["nnz"] == len(ci) and info["max_degree"] == deg.max()
    assert info["heavy_rows"] == int((deg > info["chunk"]).sum()) > 0
    assert info["heavy_chunks"] == int(np.ceil(deg[deg > info["chunk"]] / info["chunk"]).sum())
    assert info["light_rows"] + info["heavy_rows"] == w.n
    # short rows (degree <= short_max) are a subset of the light rows
    assert info["short_max"] == 32
    assert info["short_rows"] == int((deg <= info["short_max"]).sum()) > 0


@pytest.mark.parametrize("short", ["0", "4", "32"])
def test_short_row_split_parity(short):
    """The short-row kernels (4 rows per warp) against the oracle for several
    thresholds (0 = every light row through the warp-per-row kernels)."""
    opts = {"short_edges": int(short)}
    for prec in ("fp32", "bf16"):
        w = W("gat", "kron", 14, 8, 128, heads=4, act="none", prec=prec)
        src, dst, rp, ci = pu.host_graph(w)
        g = pu.device_graph(w, src, dst)
        H, Ws, As, R = w.host_inputs()
        st = pu.gpu_step(w, graph=g, R=R, plan_options=opts)
        assert st.plan.info()["short_max"] == int(short)
        ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
        pu.compare(w, st, ref, tol=pu.TOL_FP32 if prec == "fp32" else pu.TOL_BF16)
        pu.compare_attention(w, st, ref)


# ------------------------------------------------------------------ layer parity
CASES = [
    gen.CONFIGS["C1"],                                    # GAT ER 1024, k=16
    dataclasses.replace(gen.CONFIGS["C2"], act="elu"),    # GAT Kron 2^16 ef8, k=64, 2 layers
                                                          # (ELU: C1 sigma' across layers, A6')
    W("gat", "kron", 15, 8, 128, heads=4),                # C5 shape (k=128, 4 heads), heavy rows
    # factored k'=128 path with 1 / 2 / 8 heads.  The LeakyReLU branch of each entry
    # (s_i + t_j > 0, reading A5) is a floating-point decision: these inputs keep
    # min |s_i + t_j| >= 1e-6 rms(s + t) on every layer (checked with the oracle),
    # so fp32 and fp64 take the same branches (e.g. rmat 2^13 ef16 h2 has an entry
    # at 4e-7 rms; its branch flips and moves dH by 5e-4, in either GPU path)
    W("gat", "kron", 14, 8, 128, heads=1, act="elu"),
    W("gat", "rmat", 12, 16, 128, heads=2, layers=2, act="elu"),
    W("gat", "er", 0, 0, 128, heads=8, n=3000, samples=30000, act="none"),
    W("gat", "kron", 13, 8, 32, heads=8, act="elu"),
    W("gat", "er", 0, 0, 256, heads=2, n=2000, samples=12000, act="none"),
    W("gat", "rmat", 14, 8, 64, heads=1, layers=2, act="elu"),
    W("gat", "kron", 14, 8, 64, heads=2, layers=2, act="none"),
    W("agnn", "rmat", 14, 16, 128, layers=2, act="elu"),  # C3 shape (R-MAT, k=128)
    W("agnn", "kron", 13, 8, 64, act="elu"),
    W("agnn", "kron", 16, 8, 128, act="none", beta=0.7),  # k=128 kernels, heavy rows, beta != 1
    W("agnn", "er", 0, 0, 256, n=1500, samples=9000, act="none", beta=1.5),
    W("agnn", "er", 0, 0, 16, n=1024, samples=7680),
    W("va", "kron", 13, 8, 256, act="none"),              # C4 shape (VA, k=256)
    W("va", "kron", 14, 8, 128),
    W("va", "er", 0, 0, 32, n=1024, samples=7680, act="elu"),
]


@pytest.mark.parametrize("w", CASES, ids=lambda w: w.name)
def test_layer_parity(w):
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    np.testing.assert_array_equal(g.col_idx.cpu().numpy(), ci)
    H, Ws, As, R = w.host_inputs()
    if w.act == "relu":
        assert w.layers == 1, "multi-layer ReLU backward has inner-layer kink decisions (A6')"
        f0 = pu.oracle_step(dataclasses.replace(w), rp, ci, H, Ws, As, R)["fwd"][-1]
        R = pu.relu_kink_mask(w, f0["Z"], R)
    st = pu.gpu_step(w, graph=g, R=R)
    np.testing.assert_array_equal(st.H[0].cpu().numpy(), H)
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)
    pu.compare_attention(w, st, ref)


@pytest.mark.parametrize("k,heads", [(64, 2), (128, 4)])
def test_inference_mode_matches_training_forward(k, heads):
    """k' = 128 runs a different kernel variant in training (it also accumulates Q,
    the factored backward); the layer output must not change by a bit."""
    w = W("gat", "kron", 13, 8, k, heads=heads)
    st = runner.Stack(w, "cuda")
    st.forward()
    out_train = st.H[1].clone()
    st.H[1].zero_()
    st.forward(inference=True)
    torch.cuda.synchronize()
    assert torch.equal(out_train, st.H[1])


@pytest.mark.parametrize("model", ["gat", "agnn", "va"])
def test_run_to_run_bitwise_determinism(model):
    w = W(model, "kron", 14, 8, 128, heads=4 if model == "gat" else 1)
    st = runner.Stack(w, "cuda")
    st.step()
    a = [t.clone() for t in (st.H[1], st.dH[0], st.dW[0])]
    st.step()
    torch.cuda.synchronize()
    for x, y in zip(a, (st.H[1], st.dH[0], st.dW[0])):
        assert torch.equal(x, y)


def test_empty_rows_and_no_self_loops():
    """Rows without stored entries give zero output / gradient (reading A7)."""
    n, k = 50, 16
    rng = np.random.default_rng(3)
    A = rng.random((n, n)) < 0.1
    A = A | A.T
    np.fill_diagonal(A, False)
    A[7, :] = A[:, 7] = False      # isolated vertex, empty row
    rp = np.concatenate([[0], np.cumsum(A.sum(1))]).astype(np.int64)
    ci = np.concatenate([np.nonzero(A[i])[0] for i in range(n)]).astype(np.int32)
    for model, heads, kk in (("gat", 2, k), ("gat", 4, 128), ("agnn", 1, k), ("va", 1, k)):
        w = gen.Workload("edge", model, "er", 0, n, 0, kk, heads, 1, act="none")
        g = runner.Graph(n, torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), len(ci))
        st = pu.gpu_step(w, graph=g)
        H, Ws, As, R = w.host_inputs()
        ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
        pu.compare(w, st, ref)
        assert torch.all(st.H[1][7] == 0) and torch.all(st.dH[0][7] == 0)


@pytest.mark.parametrize("bad", ["unsorted", "duplicate", "range", "rowptr"])
def test_invalid_csr_rejected_at_plan(bad):
    rp = np.array([0, 2, 4, 6], np.int64)
    ci = np.array([0, 1, 0, 2, 1, 2], np.int32)
    if bad == "unsorted":
        ci[[2, 3]] = ci[[3, 2]]
    elif bad == "duplicate":
        ci[3] = 0
    elif bad == "range":
        ci[5] = 3
    else:
        rp[2] = 1
    with pytest.raises(agnn.AgnnError) as e:
        agnn.Plan(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), 3)
    assert e.value.status == 1


def test_launch_count_increases():
    w = gen.CONFIGS["C1"]
    st = runner.Stack(w, "cuda")
    c0 = agnn.launch_count()
    st.step()
    assert agnn.launch_count() > c0


# ------------------------------------------------------------------ directed patterns (A4)
DIRECTED_FLAGS = agnn.BUILD_SELF_LOOPS | agnn.BUILD_CONNECT_ISOLATED


def _directed_graph(w):
    src, dst = w.host_edges()
    rp, ci = oracle.csr_build(w.n, src, dst, flags=DIRECTED_FLAGS)
    s = torch.from_numpy(src.view(np.int32)).cuda()
    d = torch.from_numpy(dst.view(np.int32)).cuda()
    drp, dci = agnn.csr_build(w.n, s, d, DIRECTED_FLAGS)
    np.testing.assert_array_equal(drp.cpu().numpy(), rp)
    np.testing.assert_array_equal(dci.cpu().numpy(), ci)
    return rp, ci, runner.Graph(w.n, drp, dci, int(dci.numel()))


def test_plan_csc_bit_exact():
    """agnn_plan_csc: the transposed pattern + CSR positions, against a host sort."""
    w = W("gat", "kron", 14, 8, 16)
    rp, ci, g = _directed_graph(w)
    plan = agnn.Plan(g.row_ptr, g.col_idx, w.n, symmetric=False)
    cp, ri, perm = plan.csc()
    rows = np.repeat(np.arange(w.n, dtype=np.int64), np.diff(rp))
    order = np.lexsort((rows, ci))  # by column, then row
    np.testing.assert_array_equal(perm.cpu().numpy(), order)
    np.testing.assert_array_equal(ri.cpu().numpy(), rows[order].astype(np.int32))
    np.testing.assert_array_equal(cp.cpu().numpy(),
                                  np.concatenate([[0], np.cumsum(np.bincount(ci, minlength=w.n))]))


DIRECTED_CASES = [
    W("gat", "kron", 15, 8, 16, heads=1, act="none"),
    W("gat", "kron", 16, 8, 128, heads=4),
    W("gat", "rmat", 14, 16, 64, heads=2, act="elu"),
    W("agnn", "kron", 15, 8, 64),
    W("agnn", "rmat", 14, 16, 128, act="elu"),
    W("va", "kron", 14, 8, 32),
    W("va", "er", 0, 0, 128, n=5000, samples=60000, act="none"),
]


@pytest.mark.parametrize("w", DIRECTED_CASES, ids=lambda w: w.name)
def test_directed_layer_parity(w):
    """Directed pattern: row pass over the CSR + column pass over the plan's CSC."""
    rp, ci, g = _directed_graph(w)
    # the pattern really is unsymmetric (in-degrees differ from out-degrees)
    cols = np.bincount(ci, minlength=w.n)
    assert not np.array_equal(cols, np.diff(rp))
    H, Ws, As, R = w.host_inputs()
    if w.act == "relu":
        f0 = pu.oracle_step(w, rp, ci, H, Ws, As, R)["fwd"][-1]
        R = pu.relu_kink_mask(w, f0["Z"], R)
    st = pu.gpu_step(w, graph=g, R=R, symmetric=False)
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)
    pu.compare_attention(w, st, ref)


def test_directed_heavy_chunks():
    """Small chunks force heavy rows AND heavy columns through the split/merge path."""
    for model, heads in (("gat", 4), ("agnn", 1), ("va", 1)):
        w = W(model, "kron", 12, 8, 64, heads=heads, act="none")
        rp, ci, g = _directed_graph(w)
        st = pu.gpu_step(w, graph=g, symmetric=False, plan_options={"chunk_edges": 64})
        assert st.plan.info()["heavy_rows"] > 0
        H, Ws, As, R = w.host_inputs()
        pu.compare(w, st, pu.oracle_step(w, rp, ci, H, Ws, As, R))


@pytest.mark.parametrize("k,opts", [(64, None), (128, None), (128, {"spmmm": 1})],
                         ids=["k64", "k128", "k128-spmmm"])
def test_agnn_eps_branch(k, opts):
    """Reading A8 on the GPU: zero rows and rows of norm < eps = 1e-12 take
    nu_i = eps (constant), with the gradient dHhat_j / eps of the oracle
    (pinned in test_oracle_pins.py::test_agnn_eps_branch)."""
    w = W("agnn", "kron", 12, 8, k, layers=1, act="elu")
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    H, Ws, As, R = w.host_inputs()
    deg = np.diff(rp)
    zero = [int(np.argmax(deg)), 5, 77]          # the hub row among them
    tiny = [300, 1001]
    H = H.copy()
    H[zero] = 0.0
    H[tiny] *= np.float32(1e-14)
    st = runner.Stack(w, "cuda", graph=g, plan_options=opts)
    st.H[0].copy_(torch.from_numpy(H))
    st.dH[1].copy_(torch.from_numpy(R))
    st.step()
    torch.cuda.synchronize()
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)
    # the branch rows carry the 1/eps-scaled gradients; check them on their own too
    pu.compare_arrays({"dH_eps": (st.dH[0].cpu().numpy()[zero + tiny], ref["dH"][0][zero + tiny]),
                       "H_eps": (st.H[1].cpu().numpy()[zero + tiny], ref["H"][1][zero + tiny])},
                      rowwise=["dH_eps", "H_eps"])
    pu.compare_attention(w, st, ref)


def test_symmetric_flag_on_directed_pattern_is_rejected():
    """A directed pattern passed as AGNN_CSR_SYMMETRIC would silently give a wrong
    backward; with AGNN_PLAN_VERIFY_SYMMETRY the plan checks A = A^T on the device
     and refuses it, while the same check accepts the symmetric
    pattern, and the directed plan of the pattern still matches the oracle."""
    w = W("gat", "kron", 12, 8, 64, heads=2, act="none")
    rp, ci, g = _directed_graph(w)
    with pytest.raises(agnn.AgnnError) as e:
        agnn.Plan(g.row_ptr, g.col_idx, w.n, symmetric=True, verify_symmetry=True)
    assert e.value.status == 1 and "not symmetric" in str(e.value)
    st = pu.gpu_step(w, graph=g, symmetric=False)
    H, Ws, As, R = w.host_inputs()
    pu.compare(w, st, pu.oracle_step(w, rp, ci, H, Ws, As, R))
    # the symmetric pattern of the same recipe passes the check, and a plan of it with
    # the flag computes the same as the directed (two-pass) plan of it
    src, dst, rps, cis = pu.host_graph(w)
    gs = pu.device_graph(w, src, dst)
    agnn.Plan(gs.row_ptr, gs.col_idx, w.n, symmetric=True, verify_symmetry=True)
    a = pu.gpu_step(w, graph=gs)
    b = pu.gpu_step(w, graph=gs, symmetric=False)
    for x, y in ((a.dH[0], b.dH[0]), (a.dW[0], b.dW[0]), (a.da[0], b.da[0])):
        assert pu.rel(x.cpu().numpy(), y.cpu().numpy()) <= 1e-6


def test_plan_rejects_partial_rows_on_one_gpu():
    """world == 1 with row_begin > 0 would gather out of range: EINVAL (agnn.h)."""
    w = W("gat", "kron", 10, 8, 64)
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    half = w.n // 2
    rp_t = g.row_ptr[half:].contiguous() - int(rp[half])
    with pytest.raises(agnn.AgnnError) as e:
        agnn.Plan(rp_t, g.col_idx[int(rp[half]):].contiguous(), w.n, row_begin=half)
    assert e.value.status == 1


@pytest.mark.parametrize("kind,k,heads", [("gat", 48, 1), ("gat", 128, 16), ("gat", 16, 8),
                                          ("va", 48, 1), ("agnn", 96, 1), ("cgnn", 80, 1)])
def test_model_rejects_widths_without_kernels(kind, k, heads):
    """(k, heads) outside the dispatch tables fail at agnn_model_create, before any launch."""
    w = W("gat", "kron", 10, 8, 64)
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    plan = agnn.Plan(g.row_ptr, g.col_idx, w.n)
    with pytest.raises(agnn.AgnnError) as e:
        agnn.Model(plan, [agnn.layer_desc(kind, k, k, heads)])
    assert e.value.status in (1, 5)


# ------------------------------------------------------------------ C-GNN over semirings (f3)
CGNN_CASES = [
    W("cgnn", "kron", 14, 8, 64, act="elu", agg="sum"),
    W("cgnn", "kron", 14, 8, 128, act="none", agg="mean"),
    W("cgnn", "rmat", 13, 16, 32, act="elu", agg="gcn"),
    W("cgnn", "kron", 15, 8, 16, act="relu", agg="max"),
    W("cgnn", "er", 0, 0, 256, n=3000, samples=30000, act="none", agg="min"),
    W("cgnn", "kron", 13, 8, 64, layers=2, act="elu", agg="gcn"),
    W("cgnn", "kron", 13, 8, 128, layers=2, act="elu", agg="max"),
]


def _cgnn_check(w, rp, ci, g, symmetric=True, plan_options=None):
    H, Ws, As, R = w.host_inputs()
    if w.act == "relu":
        f0 = pu.oracle_step(w, rp, ci, H, Ws, As, R)["fwd"][-1]
        R = pu.relu_kink_mask(w, f0["Z"], R)
    if w.agg in ("max", "min") and w.layers > 1:
        R = pu.tropical_tie_mask(w, rp, ci, pu.oracle_step(w, rp, ci, H, Ws, As, R)["H"][-2], R)
    st = pu.gpu_step(w, graph=g, R=R, symmetric=symmetric, plan_options=plan_options)
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)
    return st, ref


@pytest.mark.parametrize("w", CGNN_CASES, ids=lambda w: f"{w.name}-{w.agg}")
def test_cgnn_layer_parity(w):
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    _cgnn_check(w, rp, ci, g)


@pytest.mark.parametrize("agg", ["sum", "mean", "gcn", "max", "min"])
def test_cgnn_directed_and_heavy_chunks(agg):
    """Directed pattern (backward gathers over the CSC) with heavy rows and columns
    split into 64-edge chunks."""
    w = W("cgnn", "kron", 12, 8, 64, act="none", agg=agg)
    rp, ci, g = _directed_graph(w)
    st, _ = _cgnn_check(w, rp, ci, g, symmetric=False, plan_options={"chunk_edges": 64})
    assert st.plan.info()["heavy_rows"] > 0
