"""GPU parity of the fused SpMMM forward (Table 2 "SpMMM: a
composition of SpMM and MM"): AGNN / VA layers with
k_in = k_out = 128 run X = Psi H and Z = X W in one kernel (agnn_plan_options.spmmm
= 1; X goes to the tcgen05 MMA through shared memory).  Every output of the
fwd+bwd step is checked against the FP64 oracle at the FP32 bars of
test_gpu_parity.py (normwise 1e-5, per-row bounds), on graphs that span many
32-row tiles, heavy rows (chunk kernel + merge, then loaded by the fused kernel)
and ragged last tiles; and against the unfused path (same arithmetic, another
summation order inside the MMA: within the bar, not bitwise).
"""
from __future__ import annotations

import dataclasses

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]

import parity_utils as pu  # noqa: E402
from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner  # noqa: E402

FUSED = {"spmmm": 1}


def W(model, graph, scale, ef, k, layers=1, act="relu", n=None, samples=None, **kw):
    n = n or (1 << scale)
    return gen.Workload(f"{model}-{graph}{scale}-k{k}L{layers}-spmmm", model, graph, scale, n,
                        samples if samples is not None else ef * n, k, 1, layers, act=act, **kw)


CASES = [
    (W("agnn", "rmat", 14, 16, 128, layers=2, act="elu"), {}),          # C3 shape, 2 layers
    (W("agnn", "kron", 16, 8, 128, act="none", beta=0.7), {}),          # heavy rows (chunks)
    (W("agnn", "kron", 13, 8, 128, act="elu"), {"chunk_edges": 64}),   # many heavy rows
    (W("va", "kron", 14, 8, 128), {}),                                  # VA, ReLU
    (W("va", "er", 0, 0, 128, n=1001, samples=6000, act="elu"), {}),    # ragged last tile
    (W("agnn", "er", 0, 0, 128, n=45, samples=200, act="none"), {}),    # fewer rows than a tile
]


def _run(w, opts, fused=True):
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    H, Ws, As, R = w.host_inputs()
    if w.act == "relu":
        f0 = pu.oracle_step(dataclasses.replace(w), rp, ci, H, Ws, As, R)["fwd"][-1]
        R = pu.relu_kink_mask(w, f0["Z"], R)
    o = dict(opts, **(FUSED if fused else {"spmmm": 0}))
    st = pu.gpu_step(w, graph=g, R=R, plan_options=o)
    return st, (rp, ci, H, Ws, As, R)


@pytest.mark.parametrize("case", CASES, ids=lambda c: c[0].name + ("-c64" if c[1] else ""))
def test_spmmm_layer_parity(case):
    w, opts = case
    st, (rp, ci, H, Ws, As, R) = _run(w, opts)
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)
    pu.compare_attention(w, st, ref)


@pytest.mark.parametrize("model", ["agnn", "va"])
def test_spmmm_matches_split_path(model):
    """Fused and unfused forward compute the same products (3xTF32, K split in two
    accumulation groups); they differ only in the MMA's internal order."""
    w = W(model, "kron", 14, 8, 128, act="elu")
    a, _ = _run(w, {}, fused=True)
    b, _ = _run(w, {}, fused=False)
    errs = pu.compare_arrays({"H1": (a.H[1].cpu().numpy(), b.H[1].cpu().numpy().astype(np.float64)),
                              "dH0": (a.dH[0].cpu().numpy(), b.dH[0].cpu().numpy().astype(np.float64)),
                              "dW0": (a.dW[0].cpu().numpy(), b.dW[0].cpu().numpy().astype(np.float64))},
                             tol=5e-6)
    assert errs["H1"] < 1e-6


@pytest.mark.parametrize("model", ["agnn", "va"])
def test_spmmm_inference_matches_training_forward(model):
    """Inference stores neither X nor Z; the layer output must not change by a bit."""
    w = W(model, "kron", 13, 8, 128, act="elu")
    st = runner.Stack(w, "cuda", plan_options=FUSED)
    st.forward()
    out_train = st.H[1].clone()
    st.H[1].zero_()
    st.forward(inference=True)
    torch.cuda.synchronize()
    assert torch.equal(out_train, st.H[1])


def test_spmmm_directed_pattern():
    """A directed pattern (no AGNN_CSR_SYMMETRIC): the forward visits row i's stored
    entries either way; the backward runs its row and column passes."""
    from test_gpu_parity import _directed_graph
    w = W("agnn", "kron", 13, 8, 128, act="elu")
    rp, ci, g = _directed_graph(w)
    H, Ws, As, R = w.host_inputs()
    st = pu.gpu_step(w, graph=g, R=R, symmetric=False, plan_options=FUSED)
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref)


def test_spmmm_bf16_storage():
    """BF16 storage (reading B2): the gathered rows are the rounded H~; X stays fp32
    into the fused projection.  Same 1e-2 protocol as test_gpu_bf16.py."""
    w = W("agnn", "rmat", 13, 16, 128, act="none", prec="bf16")
    st, (rp, ci, H, Ws, As, R) = _run(w, {})
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    pu.compare(w, st, ref, tol=pu.TOL_BF16)


def test_spmmm_empty_rows():
    """Rows without stored entries (reading A7): X_i = 0, so Z_i = 0 and H_out_i = sigma(0)."""
    n = 70
    rng = np.random.default_rng(5)
    A = rng.random((n, n)) < 0.1
    A = A | A.T
    np.fill_diagonal(A, False)
    A[7, :] = A[:, 7] = False
    A[40, :] = A[:, 40] = False
    rp = np.concatenate([[0], np.cumsum(A.sum(1))]).astype(np.int64)
    ci = np.concatenate([np.nonzero(A[i])[0] for i in range(n)]).astype(np.int32)
    for model in ("agnn", "va"):
        w = gen.Workload("edge-sp", model, "er", 0, n, 0, 128, 1, 1, act="elu")
        g = runner.Graph(n, torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), len(ci))
        st = pu.gpu_step(w, graph=g, plan_options=FUSED)
        H, Ws, As, R = w.host_inputs()
        pu.compare(w, st, pu.oracle_step(w, rp, ci, H, Ws, As, R))
        for r in (7, 40):
            assert torch.all(st.H[1][r] == 0) and torch.all(st.dH[0][r] == 0)


def test_spmmm_option_validated():
    w = W("agnn", "er", 0, 0, 128, n=64, samples=256)
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    with pytest.raises(Exception):
        pu.gpu_step(w, graph=g, plan_options={"spmmm": 2})
