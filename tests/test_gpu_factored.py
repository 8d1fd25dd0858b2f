"""GPU tests of the factored GAT backward and of the L2 residency hints.

The factored backward (gat_args.cuh) moves the row-role sum of the
GAT backward (Eq. 6 with Psi^T) into the forward:
ds_j = G_j . Q_j with Q_j = sum_i c_ji P_i - (sum_i c_ji) Z_j, c = alpha lambda.
Its parity against the FP64 oracle is covered by every GAT k' = 128 case of
test_gpu_parity.py / test_gpu_bf16.py (it is the default path); here:
  * the unfactored path (plan option gat_factored = 0) still meets the same bar, and so do
    both short-row decompositions (row groups, bundles) for both storage types;
  * the factored path gives da1 = 0 EXACTLY when LeakyReLU is linear on every
    stored entry (the a-orientation identity of test_oracle_pins.py: each row's
    softmax is invariant to s_i), where the unfactored sum only reaches ~eps;
  * the L2 eviction hints change no bit of any output.
"""
from __future__ import annotations

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]

import parity_utils as pu  # noqa: E402
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner  # noqa: E402

def W(graph, scale, ef, heads, prec="fp32", act="relu", k=128):
    n = 1 << scale
    return gen.Workload(f"gat-{graph}{scale}-h{heads}-{prec}", "gat", graph, scale, n, ef * n, k,
                        heads, 1, act=act, prec=prec)


def _directed_case(k, opts):
    import oracle
    from paper_conf_sc_bestarglzcgssci23_b200 import agnn
    w = gen.Workload("gat-dir", "gat", "kron", 13, 1 << 13, 8 << 13, k, 2, 1, act="elu")
    flags = agnn.BUILD_SELF_LOOPS | agnn.BUILD_CONNECT_ISOLATED
    src, dst = w.host_edges()
    rp, ci = oracle.csr_build(w.n, src, dst, flags=flags)
    drp, dci = agnn.csr_build(w.n, torch.from_numpy(src.view(np.int32)).cuda(),
                              torch.from_numpy(dst.view(np.int32)).cuda(), flags)
    g = runner.Graph(w.n, drp, dci, int(dci.numel()))
    st = pu.gpu_step(w, graph=g, symmetric=False, plan_options=opts)
    H, Ws, As, R = w.host_inputs()
    pu.compare(w, st, pu.oracle_step(w, rp, ci, H, Ws, As, R))


@pytest.mark.parametrize("mode,k", [(2, 64), (0, 128), (1, 128)])
def test_directed_factored_and_unfactored(mode, k):
    """Directed patterns: factored (row pass replaced by ds = G.Q) and two-pass."""
    _directed_case(k, {"chunk_edges": 128, "gat_factored": mode})


_SYM = {}


def _sym_graph():
    if "g" not in _SYM:
        w = gen.Workload("gat-kron14-h4", "gat", "kron", 14, 1 << 14, 8 << 14, 128, 4, 1,
                         act="elu")
        src, dst, rp, ci = pu.host_graph(w)
        _SYM["g"] = (rp, ci, pu.device_graph(w, src, dst))
    return _SYM["g"]


def _run(opts, prec="fp32", check=True, k=128):
    """GAT kron 2^14, 4 heads, ELU, heavy rows (256-edge chunks) under plan options."""
    w = gen.Workload("gat-kron14-h4", "gat", "kron", 14, 1 << 14, 8 << 14, k, 4, 1, act="elu",
                     prec=prec)
    rp, ci, g = _sym_graph()
    st = pu.gpu_step(w, graph=g, plan_options=dict({"chunk_edges": 256}, **opts))
    if check:
        H, Ws, As, R = w.host_inputs()
        tol = pu.TOL_BF16 if w.prec == "bf16" else pu.TOL_FP32
        pu.compare(w, st, pu.oracle_step(w, rp, ci, H, Ws, As, R), tol=tol)
    return {"H": st.H[1].cpu().numpy(), "dH": st.dH[0].cpu().numpy(),
            "dW": st.dW[0].cpu().numpy(), "da": st.da[0].cpu().numpy()}


@pytest.mark.parametrize("prec,k", [("fp32", 128), ("bf16", 128), ("fp32", 64), ("fp32", 256)])
def test_unfactored_path_parity(prec, k):
    """k' = 128: the k128 kernels; other widths: the generic row-group kernels."""
    _run({"gat_factored": 0}, prec, k=k)


@pytest.mark.parametrize("k", [32, 64, 256])
def test_factored_generic_widths_parity(k):
    """The factored backward on the generic kernels (forward with QF, then the
    column-role pass over the symmetric CSR), heavy rows included."""
    _run({"gat_factored": 2}, "fp32", k=k)


@pytest.mark.parametrize("prec", ["fp32", "bf16"])
@pytest.mark.parametrize("bundles", [0, 2])
def test_short_row_paths_parity(prec, bundles):
    """Short rows through the row-group kernels (0) or the bundle kernels (2 = for
    both storage types; the default uses bundles for fp32 only)."""
    _run({"short_bundles": bundles}, prec)


def test_l2_hints_change_no_bit():
    a = _run({"l2_hot_mb": 0}, check=False)
    b = _run({"l2_hot_mb": 1000000}, check=False)
    c = _run({}, check=False)
    for k in a:
        assert np.array_equal(a[k], b[k]) and np.array_equal(a[k], c[k]), k


def test_plan_options_rejected_out_of_range():
    from paper_conf_sc_bestarglzcgssci23_b200 import agnn
    rp, ci, g = _sym_graph()
    for bad in ({"chunk_edges": 16}, {"short_edges": 33}, {"short_bundles": 3},
                {"gat_factored": 3}):
        with pytest.raises(agnn.AgnnError) as e:
            agnn.Plan(g.row_ptr, g.col_idx, g.n, options=bad)
        assert e.value.status == 1, bad


@pytest.mark.parametrize("prec,k", [("fp32", 128), ("bf16", 128)])
def test_factored_da1_exactly_zero_when_leaky_relu_linear(prec, k):
    """H, W, a > 0 => P, s, t > 0 => every pre-activation > 0 => ds = 0 exactly."""
    w = W("kron", 13, 8, 4, prec=prec, act="none", k=k)
    st = runner.Stack(w, "cuda")
    g = torch.Generator(device="cpu").manual_seed(7)
    st.H[0].copy_(torch.rand(st.H[0].shape, generator=g) * 0.9 + 0.1)
    st.W[0].copy_(torch.rand(st.W[0].shape, generator=g) * 0.9 + 0.1)
    st.a[0].copy_(torch.rand(st.a[0].shape, generator=g) * 0.9 + 0.1)
    st.step()
    torch.cuda.synchronize()
    d = w.k // w.heads
    da = st.da[0].cpu().numpy()
    assert np.all(da[:, :d] == 0.0), np.abs(da[:, :d]).max()
    assert np.abs(da[:, d:]).max() > 1e-3
