"""Pins for the FP64 oracle (CPU only).

Each check ties oracle/agnn_oracle.c to something other than itself:
  * the dense GLOBAL formulation + torch.autograd (tests/dense_ref.py) — the
    paper's local == global claim;
  * central finite differences of L = <R, H_out> (Eq. 2-5);
  * the paper's printed VA closed forms Eq. 7, 11, 12, 13;
  * special cases: complete graph = dense softmax attention, uniform attention =
    mean aggregation (averaging semiring), A = I for VA;
  * invariants: softmax rows sum to 1, permutation equivariance,
    multi-head = concatenation of heads (reading A10), a-orientation (da1 = 0
    when LeakyReLU is linear on every edge);
  * the 3-vertex worked example (tests/golden/worked_example.json);
  * brute force for the CSR builder and the partition bounds.
"""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import dense_ref
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "worked_example.json")


def rand_graph(n, p, rng, symmetric=True, self_loops=True):
    A = rng.random((n, n)) < p
    if symmetric:
        A = A | A.T
    if self_loops:
        np.fill_diagonal(A, True)
    rp = np.zeros(n + 1, np.int64)
    cols = []
    for i in range(n):
        c = np.nonzero(A[i])[0]
        cols.extend(c.tolist())
        rp[i + 1] = rp[i] + len(c)
    return rp, np.array(cols, np.int32)


def rand_inputs(n, k, kout, heads, rng, scale=1.0):
    H = rng.uniform(-1, 1, (n, k)) * scale
    W = rng.uniform(-1, 1, (k, kout)) / np.sqrt(k)
    a = rng.uniform(-1, 1, (heads, 2 * (kout // heads)))
    R = rng.uniform(-1, 1, (n, kout))
    return H, W, a, R


def rel(x, y):
    x, y = np.asarray(x, np.float64), np.asarray(y, np.float64)
    return np.linalg.norm(x - y) / max(np.linalg.norm(y), 1e-300)


def alpha_dense(rp, ci, alpha, n, h=None):
    D = np.zeros((n, n))
    for i in range(n):
        for p in range(rp[i], rp[i + 1]):
            D[i, ci[p]] = alpha[p] if h is None else alpha[p, h]
    return D


# ---------------------------------------------------------------- dense global
@pytest.mark.parametrize("heads", [1, 2, 4])
@pytest.mark.parametrize("kind", ["none", "relu", "elu"])
@pytest.mark.parametrize("symmetric", [True, False])
def test_gat_local_equals_global(heads, kind, symmetric):
    rng = np.random.default_rng(10 + heads)
    n, k, kout = 13, 5, 8
    rp, ci = rand_graph(n, 0.3, rng, symmetric=symmetric)
    H, W, a, R = rand_inputs(n, k, kout, heads, rng)
    f, b = oracle.layer("gat", rp, ci, H, W, a, heads, R, act=kind)
    ref = dense_ref.gat(rp, ci, H, W, a, heads, R, kind=kind)
    for h in range(heads):
        assert np.abs(alpha_dense(rp, ci, f["alpha"], n, h) - ref["Psi"][h]).max() < 1e-13
    assert rel(f["Z"], ref["Z"]) < 1e-13
    assert rel(f["Hout"], ref["Hout"]) < 1e-13
    assert rel(b["dH"], ref["dH"]) < 1e-12
    assert rel(b["dW"], ref["dW"]) < 1e-12
    assert rel(b["da"], ref["da"]) < 1e-11


@pytest.mark.parametrize("beta", [1.0, 1.3])
@pytest.mark.parametrize("kind", ["none", "relu", "elu"])
@pytest.mark.parametrize("symmetric", [True, False])
def test_agnn_local_equals_global(beta, kind, symmetric):
    rng = np.random.default_rng(20)
    n, k, kout = 12, 6, 4
    rp, ci = rand_graph(n, 0.35, rng, symmetric=symmetric)
    H, W, _, R = rand_inputs(n, k, kout, 1, rng)
    f, b = oracle.layer("agnn", rp, ci, H, W, dHout=R, act=kind, beta=beta)
    ref = dense_ref.agnn(rp, ci, H, W, R, beta=beta, kind=kind)
    assert np.abs(alpha_dense(rp, ci, f["alpha"], n) - ref["Psi"]).max() < 1e-13
    assert rel(f["X"], ref["X"]) < 1e-13
    assert rel(f["Z"], ref["Z"]) < 1e-13
    assert rel(b["dH"], ref["dH"]) < 1e-12
    assert rel(b["dW"], ref["dW"]) < 1e-12


@pytest.mark.parametrize("kind", ["none", "elu"])
@pytest.mark.parametrize("symmetric", [True, False])
def test_agnn_eps_branch(kind, symmetric):
    """Reading A8: nu_i = max(|H_i|, eps), constant on the eps branch.  A zero row and a
    row of norm ~1e-14 < eps = 1e-12 take the branch: the oracle matches autograd of
    the dense formulation with a clamped norm (torch.clamp passes no gradient below
    eps), and the closed forms of the branch hold: the zero row scores c_ij = 0, so its
    attention is uniform (mean aggregation), and its input gradient is
    exactly dHhat_j / eps (no projection term, since d(H/eps)/dH = I/eps)."""
    rng = np.random.default_rng(21)
    n, k, kout = 12, 6, 4
    rp, ci = rand_graph(n, 0.35, rng, symmetric=symmetric)
    H, W, _, R = rand_inputs(n, k, kout, 1, rng)
    H[3] = 0.0
    H[7] *= 1e-14
    assert np.linalg.norm(H[7]) < 1e-12
    f, b = oracle.layer("agnn", rp, ci, H, W, dHout=R, act=kind, beta=1.3)
    ref = dense_ref.agnn(rp, ci, H, W, R, beta=1.3, kind=kind)
    assert np.abs(alpha_dense(rp, ci, f["alpha"], n) - ref["Psi"]).max() < 1e-13
    assert rel(f["Z"], ref["Z"]) < 1e-13
    assert rel(b["dH"], ref["dH"]) < 1e-12 and rel(b["dH"][3], ref["dH"][3]) < 1e-12
    assert rel(b["dH"][7], ref["dH"][7]) < 1e-12
    assert rel(b["dW"], ref["dW"]) < 1e-12
    # zero row: uniform attention over its stored entries, X_3 = mean of its neighbours
    row = slice(rp[3], rp[4])
    np.testing.assert_allclose(f["alpha"][row], 1.0 / (rp[4] - rp[3]), rtol=1e-14)
    np.testing.assert_allclose(f["X"][3], H[ci[row]].mean(0), rtol=1e-12, atol=1e-15)
    # the branch's gradient scale: |dH_j| ~ |dHhat_j| / eps >> the other rows
    assert np.linalg.norm(b["dH"][3]) > 1e6 * np.linalg.norm(b["dH"][0])


@pytest.mark.parametrize("kind", ["none", "relu", "elu"])
@pytest.mark.parametrize("symmetric", [True, False])
def test_va_local_equals_global_and_eq11_13(kind, symmetric):
    rng = np.random.default_rng(30)
    n, k, kout = 11, 5, 7
    rp, ci = rand_graph(n, 0.3, rng, symmetric=symmetric)
    H, W, _, R = rand_inputs(n, k, kout, 1, rng)
    f, b = oracle.layer("va", rp, ci, H, W, dHout=R, act=kind)
    ref = dense_ref.va(rp, ci, H, W, R, kind=kind)
    cf = dense_ref.va_closed_form(rp, ci, H, W, R, kind=kind)
    assert rel(f["Z"], ref["Z"]) < 1e-13
    assert rel(f["Z"], cf["Z"]) < 1e-13                  # Eq. 7
    assert rel(b["dH"], ref["dH"]) < 1e-12
    assert rel(b["dH"], cf["dH"]) < 1e-12                # Eq. 11/12 Gamma
    assert rel(b["dW"], ref["dW"]) < 1e-12
    assert rel(b["dW"], cf["dW"]) < 1e-12                # Eq. 13 Y


# ------------------------------------------------------- finite differences
def _fd(fun, x, eps=1e-6):
    g = np.zeros_like(x)
    it = np.nditer(x, flags=["multi_index"])
    for _ in it:
        idx = it.multi_index
        old = x[idx]
        x[idx] = old + eps
        fp = fun()
        x[idx] = old - eps
        fm = fun()
        x[idx] = old
        g[idx] = (fp - fm) / (2 * eps)
    return g


@pytest.mark.parametrize("model", ["gat", "agnn", "va"])
@pytest.mark.parametrize("kind", ["none", "elu"])
def test_finite_differences(model, kind):
    rng = np.random.default_rng(40)
    n, k, kout, heads = 8, 4, 4, (2 if model == "gat" else 1)
    rp, ci = rand_graph(n, 0.35, rng, symmetric=(model != "va"))
    H, W, a, R = rand_inputs(n, k, kout, heads, rng)

    def loss():
        f, _ = oracle.layer(model, rp, ci, H, W, a, heads, act=kind, beta=1.1)
        return float((f["Hout"] * R).sum())

    _, b = oracle.layer(model, rp, ci, H, W, a, heads, R, act=kind, beta=1.1)
    assert rel(b["dH"], _fd(loss, H)) < 1e-7
    assert rel(b["dW"], _fd(loss, W)) < 1e-7
    if model == "gat":
        assert rel(b["da"], _fd(loss, a)) < 1e-7


# ------------------------------------------------------------ worked example
def _golden_graph():
    g = json.load(open(GOLDEN))
    rows = g["graph_rows"]
    rp = np.cumsum([0] + [len(r) for r in rows]).astype(np.int64)
    ci = np.array([c for r in rows for c in r], np.int32)
    return g, rp, ci


def test_worked_example_gat():
    g, rp, ci = _golden_graph()
    H, W, R = (np.array(g[x], float) for x in ("H", "W", "R"))
    v1 = g["gat_v1"]
    f, b = oracle.layer("gat", rp, ci, H, W, np.array(v1["a"], float), 1, R, act="none")
    np.testing.assert_allclose(f["s"][:, 0], v1["s"], atol=1e-12)
    np.testing.assert_allclose(f["t"][:, 0], v1["t"], atol=1e-12)
    np.testing.assert_allclose(f["alpha"][:, 0], [x for r in v1["alpha_rows"] for x in r], atol=1e-11)
    np.testing.assert_allclose(f["Z"], v1["Z"], atol=1e-11)
    np.testing.assert_allclose(b["dH"].ravel(), v1["dH"], atol=1e-11)
    np.testing.assert_allclose(b["dW"].ravel(), v1["dW"], atol=1e-11)
    np.testing.assert_allclose(b["da"][0, :2], v1["da1"], atol=1e-11)
    np.testing.assert_allclose(b["da"][0, 2:], v1["da2"], atol=1e-11)
    v2 = g["gat_v2"]
    f, b = oracle.layer("gat", rp, ci, H, W, np.array(v2["a"], float), 1, R, act="none")
    np.testing.assert_allclose(f["s"][:, 0], v2["s"], atol=1e-12)
    np.testing.assert_allclose(f["alpha"][2:5, 0], v2["alpha_row1"], atol=1e-11)
    np.testing.assert_allclose(f["Z"][1], v2["Z_row1"], atol=1e-11)
    np.testing.assert_allclose(b["dH"].ravel(), v2["dH"], atol=1e-11)
    np.testing.assert_allclose(b["dW"].ravel(), v2["dW"], atol=1e-11)
    np.testing.assert_allclose(b["da"][0, :2], v2["da1"], atol=1e-11)
    np.testing.assert_allclose(b["da"][0, 2:], v2["da2"], atol=1e-11)


def test_worked_example_agnn_va():
    g, rp, ci = _golden_graph()
    H, W, R = (np.array(g[x], float) for x in ("H", "W", "R"))
    f, b = oracle.layer("agnn", rp, ci, H, W, dHout=R, act="none")
    np.testing.assert_allclose(f["alpha"], [x for r in g["agnn"]["alpha_rows"] for x in r], atol=1e-11)
    np.testing.assert_allclose(f["Z"], g["agnn"]["Z"], atol=1e-11)
    np.testing.assert_allclose(b["dH"].ravel(), g["agnn"]["dH"], atol=1e-11)
    np.testing.assert_allclose(b["dW"].ravel(), g["agnn"]["dW"], atol=1e-11)
    f, b = oracle.layer("va", rp, ci, H, W, dHout=R, act="none")
    np.testing.assert_allclose(alpha_dense(rp, ci, f["S"], 3), g["va"]["S_dense"], atol=0)
    np.testing.assert_allclose(f["Z"], g["va"]["Z"], atol=0)
    np.testing.assert_allclose(b["dH"].ravel(), g["va"]["dH"], atol=0)
    np.testing.assert_allclose(b["dW"].ravel(), g["va"]["dW"], atol=0)


# ------------------------------------------------------------ special cases
def test_complete_graph_is_dense_softmax_attention():
    rng = np.random.default_rng(50)
    n, k, heads = 7, 4, 1
    rp = np.arange(0, n * n + 1, n, dtype=np.int64)
    ci = np.tile(np.arange(n, dtype=np.int32), n)
    H, W, a, _ = rand_inputs(n, k, k, heads, rng)
    f, _ = oracle.layer("gat", rp, ci, H, W, a, heads, act="none")
    P = H @ W
    C = (P @ a[0, :k])[:, None] + (P @ a[0, k:])[None, :]
    E = np.where(C > 0, C, 0.2 * C)
    S = np.exp(E - E.max(1, keepdims=True))
    S /= S.sum(1, keepdims=True)
    assert rel(f["Z"], S @ P) < 1e-13
    f, _ = oracle.layer("agnn", rp, ci, H, W, act="none")
    Hn = H / np.linalg.norm(H, axis=1, keepdims=True)
    C = Hn @ Hn.T
    S = np.exp(C - C.max(1, keepdims=True))
    S /= S.sum(1, keepdims=True)
    assert rel(f["Z"], S @ H @ W) < 1e-13


def test_uniform_attention_is_mean_aggregation():
    """Averaging semiring: uniform alpha => Z = D^-1 A H W."""
    rng = np.random.default_rng(60)
    n, k = 15, 6
    rp, ci = rand_graph(n, 0.3, rng)
    H, W, a, _ = rand_inputs(n, k, k, 2, rng)
    A = dense_ref.dense_mask(rp, ci, n).numpy().astype(float)
    Dinv = 1.0 / A.sum(1, keepdims=True)
    f, _ = oracle.layer("gat", rp, ci, H, W, np.zeros_like(a), 2, act="none")
    assert rel(f["Z"], (Dinv * A) @ H @ W) < 1e-13
    v = rng.uniform(0.5, 1, k)
    Hpar = rng.uniform(0.5, 2, (n, 1)) * v[None, :]           # all rows parallel: cos = 1
    f, _ = oracle.layer("agnn", rp, ci, Hpar, W, act="none")
    assert rel(f["Z"], (Dinv * A) @ Hpar @ W) < 1e-13
    f, _ = oracle.layer("agnn", rp, ci, H, W, act="none", beta=0.0)  # beta -> 0
    assert rel(f["Z"], (Dinv * A) @ H @ W) < 1e-13


def test_va_identity_graph():
    rng = np.random.default_rng(70)
    n, k = 9, 5
    rp = np.arange(n + 1, dtype=np.int64)
    ci = np.arange(n, dtype=np.int32)
    H, W, _, _ = rand_inputs(n, k, k, 1, rng)
    f, _ = oracle.layer("va", rp, ci, H, W, act="none")
    assert rel(f["Z"], (np.sum(H * H, 1, keepdims=True) * H) @ W) < 1e-14


def test_rows_sum_to_one_and_positive():
    rng = np.random.default_rng(80)
    n = 30
    rp, ci = rand_graph(n, 0.2, rng)
    H, W, a, _ = rand_inputs(n, 8, 8, 4, rng)
    f, _ = oracle.layer("gat", rp, ci, H, W, a, 4)
    g, _ = oracle.layer("agnn", rp, ci, H, W)
    for i in range(n):
        sl = slice(rp[i], rp[i + 1])
        np.testing.assert_allclose(f["alpha"][sl].sum(0), 1.0, atol=1e-14)
        np.testing.assert_allclose(g["alpha"][sl].sum(), 1.0, atol=1e-14)
    assert (f["alpha"] > 0).all() and (g["alpha"] > 0).all()


@pytest.mark.parametrize("model", ["gat", "agnn", "va"])
def test_permutation_equivariance(model):
    rng = np.random.default_rng(90)
    n, k, heads = 14, 4, (2 if model == "gat" else 1)
    rp, ci = rand_graph(n, 0.3, rng)
    H, W, a, R = rand_inputs(n, k, k, heads, rng)
    perm = rng.permutation(n)               # new id of old vertex v is perm[v]
    inv = np.argsort(perm)
    A = dense_ref.dense_mask(rp, ci, n).numpy()
    Ap = A[np.ix_(inv, inv)]
    rp2 = np.concatenate([[0], np.cumsum(Ap.sum(1))]).astype(np.int64)
    ci2 = np.concatenate([np.nonzero(Ap[i])[0] for i in range(n)]).astype(np.int32)
    f1, b1 = oracle.layer(model, rp, ci, H, W, a, heads, R)
    f2, b2 = oracle.layer(model, rp2, ci2, H[inv], W, a, heads, R[inv])
    assert rel(f2["Z"], f1["Z"][inv]) < 1e-13
    assert rel(b2["dH"], b1["dH"][inv]) < 1e-12
    assert rel(b2["dW"], b1["dW"]) < 1e-12


def test_multihead_is_concatenation():
    rng = np.random.default_rng(100)
    n, k, kout, heads = 16, 6, 8, 4
    d = kout // heads
    rp, ci = rand_graph(n, 0.25, rng)
    H, W, a, R = rand_inputs(n, k, kout, heads, rng)
    f, b = oracle.layer("gat", rp, ci, H, W, a, heads, R, act="none")
    dH = np.zeros_like(H)
    for h in range(heads):
        sl = slice(h * d, (h + 1) * d)
        fh, bh = oracle.layer("gat", rp, ci, H, W[:, sl], a[h:h + 1], 1, R[:, sl], act="none")
        assert rel(f["Z"][:, sl], fh["Z"]) < 1e-14
        assert rel(b["dW"][:, sl], bh["dW"]) < 1e-13
        assert rel(b["da"][h], bh["da"][0]) < 1e-13
        dH += bh["dH"]
    assert rel(b["dH"], dH) < 1e-13


def test_a_orientation_da1_vanishes_when_leaky_relu_is_linear():
    """If every s_i + t_j > 0, each row's softmax is invariant to s_i => da1 = 0."""
    rng = np.random.default_rng(110)
    n, k = 12, 4
    rp, ci = rand_graph(n, 0.3, rng)
    H = rng.uniform(0.1, 1, (n, k))
    W = rng.uniform(0.1, 1, (k, k))
    a = rng.uniform(0.1, 1, (1, 2 * k))
    R = rng.uniform(-1, 1, (n, k))
    f, b = oracle.layer("gat", rp, ci, H, W, a, 1, R, act="none")
    assert (f["s"][:, 0][:, None] + f["t"][:, 0][None, :] > 0).all()
    assert np.abs(b["da"][0, :k]).max() < 1e-12
    assert np.abs(b["da"][0, k:]).max() > 1e-3
    b2 = oracle.gat_backward(rp, ci, H, W, a[:, ::-1].copy(), 1,
                             oracle.gat_forward(rp, ci, H, W, a[:, ::-1].copy(), 1, act="none"),
                             R, act="none")
    assert np.abs(b2["da"][0, :k]).max() < 1e-12      # still the centre half that vanishes
    assert np.abs(b2["da"][0, k:]).max() > 1e-3


def test_empty_row_gives_zero_output_and_gradient():
    n, k = 4, 3
    rp = np.array([0, 2, 4, 4, 5], np.int64)       # row 2 has no stored entries
    ci = np.array([0, 1, 0, 1, 3], np.int32)
    rng = np.random.default_rng(120)
    H, W, a, R = rand_inputs(n, k, k, 1, rng)
    for model in ("gat", "agnn", "va"):
        f, b = oracle.layer(model, rp, ci, H, W, a, 1, R, act="none")
        assert np.all(f["Z"][2] == 0)
        assert np.all(b["dH"][2] == 0)


# ------------------------------------------------------- CSR + partition
def brute_csr(n, src, dst, flags):
    E = set()
    for s, d in zip(src.tolist(), dst.tolist()):
        if s == d:
            continue
        E.add((s, d))
        if flags & 1:
            E.add((d, s))
    if flags & 4 and n > 1:
        has = {s for s, _ in E}
        for v in range(n):
            if v not in has:
                E.add((v, (v + 1) % n))
                E.add(((v + 1) % n, v))
    if flags & 2:
        E |= {(v, v) for v in range(n)}
    E = sorted(E)
    rp = np.zeros(n + 1, np.int64)
    for s, _ in E:
        rp[s + 1] += 1
    return np.cumsum(rp), np.array([d for _, d in E], np.int32)


@pytest.mark.parametrize("flags", [0, 1, 3, 7, 5])
def test_csr_build_bruteforce(flags):
    rng = np.random.default_rng(130 + flags)
    for n in (1, 2, 5, 33, 64):
        m = int(rng.integers(0, 3 * n + 1))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        rp, ci = oracle.csr_build(n, src, dst, flags)
        rp2, ci2 = brute_csr(n, src, dst, flags)
        np.testing.assert_array_equal(rp, rp2)
        np.testing.assert_array_equal(ci, ci2)


def brute_bounds(rp, world, c_v):
    n = len(rp) - 1
    w = [int(rp[r]) + c_v * r for r in range(n + 1)]
    b = [0]
    for p in range(1, world):
        target = -(-p * w[n] // world)
        b.append(min([r for r in range(n + 1) if w[r] >= target] + [n]))
    return np.array(b + [n], np.int64)


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("c_v", [0, 4])
def test_partition_bruteforce(world, c_v):
    rng = np.random.default_rng(140 + world)
    for n in (0, 1, 7, 100):
        deg = rng.integers(0, 20, n)
        rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
        b = oracle.partition(rp, world, c_v)
        np.testing.assert_array_equal(b, brute_bounds(rp, world, c_v))
        assert (np.diff(b) >= 0).all()


# ------------------------------------------------ C-GNN over semirings (f3)
def _dense_adj(rp, ci, n):
    A = np.zeros((n, n))
    for i in range(n):
        A[i, ci[rp[i]:rp[i + 1]]] = 1.0
    return A


def _cgnn_dense_torch(A, H, W, R, agg, kind):
    """sigma(A' H W) with A' the (normalised) adjacency, or the
    tropical max/min product, in torch fp64 with autograd."""
    import torch
    At = torch.tensor(A)
    Ht = torch.tensor(H, requires_grad=True)
    Wt = torch.tensor(W, requires_grad=True)
    d = At.sum(1)
    if agg == "sum":
        X = At @ Ht
    elif agg == "mean":
        X = (At / d[:, None]) @ Ht
    elif agg == "gcn":
        X = (At / torch.sqrt(d[:, None] * d[None, :])) @ Ht
    else:
        big = torch.where(At[:, :, None] > 0, Ht[None, :, :],
                          torch.tensor(-np.inf if agg == "max" else np.inf, dtype=torch.float64))
        X = big.amax(1) if agg == "max" else big.amin(1)
    Z = X @ Wt
    Hout = {"none": Z, "relu": torch.relu(Z), "elu": torch.nn.functional.elu(Z)}[kind]
    (Hout * torch.tensor(R)).sum().backward()
    return X.detach().numpy(), Z.detach().numpy(), Ht.grad.numpy(), Wt.grad.numpy()


@pytest.mark.parametrize("agg", ["sum", "mean", "gcn", "max", "min"])
@pytest.mark.parametrize("kind", ["none", "elu"])
@pytest.mark.parametrize("symmetric", [True, False])
def test_cgnn_local_equals_dense_semiring(agg, kind, symmetric):
    """Local edge loops == the dense matrix product over the semiring + autograd.
    Features are distinct per column (no ties), so amax/amin autograd is exact."""
    rng = np.random.default_rng(60)
    n, k, kout = 14, 5, 6
    rp, ci = rand_graph(n, 0.3, rng, symmetric=symmetric)
    H = rng.permutation(n * k).reshape(n, k) / (n * k) - 0.5   # distinct values
    W = rng.uniform(-1, 1, (k, kout)) / np.sqrt(k)
    R = rng.uniform(-1, 1, (n, kout))
    f, b = oracle.layer("cgnn", rp, ci, H, W, dHout=R, act=kind, agg=agg)
    X, Z, dH, dW = _cgnn_dense_torch(_dense_adj(rp, ci, n), H, W, R, agg, kind)
    assert rel(f["X"], X) < 1e-14
    assert rel(f["Z"], Z) < 1e-13
    assert rel(b["dH"], dH) < 1e-12
    assert rel(b["dW"], dW) < 1e-12


def test_cgnn_mean_equals_paper_tuple_semiring():
    """the averaging aggregation as a product over R^2 with
    a op1 b = (a1 b1, a1) and a op2 b = ((a1 a2 + b1 b2)/(a2 + b2), a2 + b2),
    every stored entry x of A mapped to (x, x) — evaluated literally."""
    rng = np.random.default_rng(61)
    n, k = 12, 4
    rp, ci = rand_graph(n, 0.3, rng, symmetric=False)
    H = rng.uniform(-1, 1, (n, k))
    W = np.eye(k)
    f = oracle.cgnn_forward(rp, ci, H, W, "mean", "none")
    for i in range(n):
        for c in range(k):
            acc = None
            for p in range(rp[i], rp[i + 1]):
                a = (1.0, 1.0)                          # entry x = 1 -> (x, x)
                prod = (a[0] * H[ci[p], c], a[0])       # op1 with (h, .)
                acc = prod if acc is None else (
                    (acc[0] * acc[1] + prod[0] * prod[1]) / (acc[1] + prod[1]), acc[1] + prod[1])
            assert abs(f["X"][i, c] - acc[0]) < 1e-14


def test_cgnn_tropical_ties_and_empty_rows():
    """Readings C3/C4: an empty row aggregates to 0 with zero gradient; among tied
    maxima the smallest column index receives the whole gradient."""
    n, k = 4, 1
    rp = np.array([0, 3, 3, 4, 5], np.int64)        # row 1 empty
    ci = np.array([0, 2, 3, 2, 3], np.int32)
    H = np.array([[0.5], [9.0], [0.5], [0.5]])      # row 0: H_0 = H_2 = H_3 (tie)
    W = np.eye(1)
    R = np.array([[1.0], [1.0], [1.0], [1.0]])
    for agg in ("max", "min"):
        f = oracle.cgnn_forward(rp, ci, H, W, agg, "none")
        b = oracle.cgnn_backward(rp, ci, H, W, f, R, agg, "none")
        assert f["X"][1, 0] == 0.0 and f["arg"][0, 0] == 0
        # dH_0 gets row 0's gradient (first of the tie); rows 2, 3 get their own rows'
        np.testing.assert_array_equal(b["dH"][:, 0], [1.0, 0.0, 1.0, 1.0])


@pytest.mark.parametrize("agg", ["sum", "gcn", "max"])
def test_cgnn_finite_differences(agg):
    rng = np.random.default_rng(62)
    n, k, kout = 9, 3, 4
    rp, ci = rand_graph(n, 0.35, rng, symmetric=True)
    H = rng.permutation(n * k).reshape(n, k) / (n * k) - 0.5
    W = rng.uniform(-1, 1, (k, kout))
    R = rng.uniform(-1, 1, (n, kout))
    f, b = oracle.layer("cgnn", rp, ci, H, W, dHout=R, act="elu", agg=agg)
    loss = lambda: float((oracle.cgnn_forward(rp, ci, H, W, agg, "elu")["Hout"] * R).sum())
    assert rel(_fd(loss, H, 1e-7), b["dH"]) < 1e-6
    assert rel(_fd(loss, W, 1e-7), b["dW"]) < 1e-6


# ------------------------------------------------ BF16 storage mode (reading B1)
def test_bf16_round_matches_torch():
    """The oracle's bf16 rounding == torch's fp32 -> bfloat16 conversion (RNE)."""
    import torch
    rng = np.random.default_rng(70)
    x = np.concatenate([rng.standard_normal(10000) * 10.0 ** rng.integers(-30, 30, 10000),
                        [0.0, -0.0, 1.0, 1.00390625, 1.0 + 2 ** -9, 3.0e38]])
    rp = np.arange(len(x) + 1, dtype=np.int64)
    ci = np.arange(len(x), dtype=np.int32)
    # P = H W with W = 1 (k = kout = 1): the stored P~ is round_bf16(fp32(x))
    f = oracle.gat_forward(rp, ci, x[:, None], np.ones((1, 1)), np.zeros((1, 2)), 1,
                           act="none", bf16=True)
    ref = torch.tensor(x, dtype=torch.float64).float().bfloat16().double().numpy()
    np.testing.assert_array_equal(f["P"][:, 0], ref)


@pytest.mark.parametrize("heads", [1, 2])
def test_bf16_mode_exact_when_representable(heads):
    """When P and G are bf16-representable the BF16 mode IS the fp64 oracle (the
    rounding is the only difference): small-integer H, W, R and sigma = identity."""
    rng = np.random.default_rng(71)
    n, k, kout = 10, 3, 4
    rp, ci = rand_graph(n, 0.4, rng)
    H = rng.integers(-2, 3, (n, k)).astype(float)
    W = rng.integers(-2, 3, (k, kout)).astype(float)
    a = rng.uniform(-0.5, 0.5, (heads, 2 * (kout // heads)))
    R = rng.integers(-2, 3, (n, kout)).astype(float)
    f0, b0 = oracle.layer("gat", rp, ci, H, W, a, heads, R, act="none")
    f1, b1 = oracle.layer("gat", rp, ci, H, W, a, heads, R, act="none", bf16=True)
    for key in ("P", "Z", "alpha"):
        np.testing.assert_array_equal(f0[key], f1[key])
    for key in ("dH", "dW", "da"):
        np.testing.assert_array_equal(b0[key], b1[key])


def test_bf16_mode_within_the_north_star_bound():
    """Against the fp64 oracle the BF16 mode stays within the 1e-2 (north_star)."""
    rng = np.random.default_rng(72)
    n, k, kout, heads = 30, 8, 8, 2
    rp, ci = rand_graph(n, 0.3, rng)
    H, W, a, R = rand_inputs(n, k, kout, heads, rng)
    f0, b0 = oracle.layer("gat", rp, ci, H, W, a, heads, R, act="elu")
    f1, b1 = oracle.layer("gat", rp, ci, H, W, a, heads, R, act="elu", bf16=True)
    assert 0 < rel(f1["Z"], f0["Z"]) < 1e-2
    for key in ("dH", "dW"):
        assert 0 < rel(b1[key], b0[key]) < 1e-2


@pytest.mark.parametrize("model", ["agnn", "va"])
def test_agnn_va_bf16_mode_exact_when_representable(model):
    """Reading B2 (AGNN / VA BF16 storage): the mode computes the fp64 layer on
    H~ = bf16(H) with M~ = bf16(G W^T).  With H and M bf16-representable (H in
    {-1, 0, 1}, W and R on a 2^-3 grid, act none, so G = R and M = R W^T lands on
    the 2^-6 grid below 2^8) both roundings are exact and the mode IS the fp64 oracle."""
    rng = np.random.default_rng(41)
    n, k = 14, 8
    rp, ci = rand_graph(n, 0.3, rng)
    H = rng.integers(-1, 2, (n, k)).astype(np.float64)
    W = rng.integers(-2, 3, (k, k)) * 0.125
    R = rng.integers(-2, 3, (n, k)) * 0.125
    f0, b0 = oracle.layer(model, rp, ci, H, W, dHout=R, act="none")
    f1, b1 = oracle.layer(model, rp, ci, H, W, dHout=R, act="none", bf16=True)
    for x, y in ((f0["Z"], f1["Z"]), (b0["dH"], b1["dH"]), (b0["dW"], b1["dW"])):
        np.testing.assert_array_equal(x, y)


@pytest.mark.parametrize("model", ["agnn", "va"])
def test_agnn_va_bf16_mode_rounds_and_stays_within_bound(model):
    """Generic inputs: the mode differs from the unrounded oracle (the rounding is
    real) by far less than north_star's 1e-2, and equals the unrounded oracle run on
    the rounded input H~ in the forward (only M's rounding is inside the backward)."""
    rng = np.random.default_rng(42)
    n, k = 16, 8
    rp, ci = rand_graph(n, 0.3, rng)
    H, W, _, R = rand_inputs(n, k, k, 1, rng)
    f0, b0 = oracle.layer(model, rp, ci, H, W, dHout=R, act="elu")
    f1, b1 = oracle.layer(model, rp, ci, H, W, dHout=R, act="elu", bf16=True)
    fr, _ = oracle.layer(model, rp, ci, oracle.bf16_round(H), W, act="elu")
    np.testing.assert_array_equal(f1["Z"], fr["Z"])
    assert 1e-6 < rel(b1["dH"], b0["dH"]) < 1e-2
    assert 1e-6 < rel(f1["Z"], f0["Z"]) < 1e-2
