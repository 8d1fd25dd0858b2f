"""The steps either side of the layer path: loss (reading A13),
SGD update and a multi-step, multi-layer training loop, all through
the C ABI, against the FP64 oracle driving the same loop."""
from __future__ import annotations

import dataclasses

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]

import parity_utils as pu  # noqa: E402
from paper_conf_sc_bestarglzcgssci23_b200 import agnn, gen, runner  # noqa: E402


@pytest.mark.parametrize("count", [0, 1, 7, 4096, 1 << 20, (1 << 20) + 3])
def test_loss_inner_exact_fp64(count):
    g = torch.Generator().manual_seed(count)
    R = torch.rand(max(count, 1), generator=g)[:count].cuda()
    H = torch.rand(max(count, 1), generator=g)[:count].cuda()
    scratch = torch.empty(agnn.LOSS_SCRATCH, dtype=torch.float64, device="cuda")
    out = torch.full((1,), np.nan, dtype=torch.float64, device="cuda")
    agnn.loss_inner(R, H, scratch, out)
    ref = float(np.dot(R.cpu().double().numpy(), H.cpu().double().numpy()))
    got = float(out.item())
    assert abs(got - ref) <= 1e-13 * max(1.0, abs(ref)), (got, ref)
    out2 = torch.empty_like(out)
    agnn.loss_inner(R, H, scratch, out2)
    assert float(out2.item()) == got  # fixed reduction order


def test_sgd_step():
    g = torch.Generator().manual_seed(3)
    W = torch.randn(1000, 37, generator=g)
    dW = torch.randn(1000, 37, generator=g)
    Wd = W.cuda()
    agnn.sgd_step(Wd, dW.cuda(), 0.125)
    ref = W.double() - 0.125 * dW.double()   # lr a power of two: exact up to one rounding
    np.testing.assert_array_equal(Wd.cpu().numpy(), ref.float().numpy())


@pytest.mark.parametrize("model,heads", [("gat", 2), ("agnn", 1), ("va", 1)])
def test_training_loop_matches_oracle(model, heads):
    """3 SGD steps of a 2-layer model: the weights after each step and the losses
    track the oracle-driven loop (same inputs, same lr)."""
    w = dataclasses.replace(gen.Workload(f"train-{model}", model, "kron", 12, 1 << 12, 8 << 12,
                                         32, heads, 2, act="elu", beta=1.3 if model == "agnn" else 1.0),
                            train=True, lr=1e-3)
    src, dst, rp, ci = pu.host_graph(w)
    g = pu.device_graph(w, src, dst)
    st = runner.Stack(w, "cuda", graph=g)
    H, Ws, As, R = w.host_inputs()
    if model == "va":  # reading A9: multi-layer VA inputs scaled by 1/sqrt(k)
        H = H / np.sqrt(w.k)
        st.H[0].copy_(torch.from_numpy(H.astype(np.float32)))
    Ws = [x.astype(np.float64) for x in Ws]
    As = [None if x is None else x.astype(np.float64) for x in As]
    for it in range(3):
        st.step()
        loss = float(st.loss().item())
        ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
        ref_loss = float(np.sum(ref["H"][-1] * R))
        assert abs(loss - ref_loss) <= 1e-5 * np.linalg.norm(ref["H"][-1]) * np.linalg.norm(R), it
        for l in range(w.layers):
            Ws[l] = Ws[l] - w.lr * ref["dW"][l]
            if As[l] is not None:
                As[l] = As[l] - w.lr * ref["da"][l]
            assert pu.rel(st.W[l].cpu().numpy(), Ws[l]) <= pu.TOL_FP32, (it, l)
            if As[l] is not None:
                assert pu.rel(st.a[l].cpu().numpy(), As[l]) <= pu.TOL_FP32, (it, l)
