"""Dense GLOBAL formulations of one A-GNN layer in plain PyTorch fp64 (CPU).

Independent pin for the oracle (which is the edge-by-edge LOCAL form): the
paper's central claim is that local and global formulations coincide
(PAPER.md:77-83, :173-177, :191, :211).  Here the n x n virtual matrices are
built explicitly (fine for n <= ~64), the softmax is the masked global
sm(X) = exp(X) (/) rs_n(exp(X)) over the non-zeros, and
every gradient comes from torch.autograd of L = <R, H_out> (reading A13), not
from a hand-derived formula.
"""
from __future__ import annotations

import numpy as np
import torch

DT = torch.float64


def dense_mask(rp, ci, n):
    A = torch.zeros((n, n), dtype=torch.bool)
    for i in range(n):
        for p in range(rp[i], rp[i + 1]):
            A[i, ci[p]] = True
    return A


def act(z, kind):
    if kind == "relu":
        return torch.relu(z)
    if kind == "elu":
        return torch.nn.functional.elu(z)
    return z


def masked_softmax(C, A):
    """sm over the stored entries of each row; rows without entries give 0."""
    X = torch.where(A, C, torch.full_like(C, -torch.inf))
    mx = X.max(dim=1, keepdim=True).values
    mx = torch.where(torch.isfinite(mx), mx, torch.zeros_like(mx))
    E = torch.where(A, torch.exp(X - mx), torch.zeros_like(C))
    den = E.sum(dim=1, keepdim=True)
    return E / torch.where(den > 0, den, torch.ones_like(den))


def _t(x, grad=False):
    return torch.tensor(np.asarray(x, dtype=np.float64), dtype=DT, requires_grad=grad)


def gat(rp, ci, H, W, a, heads, R=None, slope=0.2, kind="relu"):
    """Psi = sm(A (.) sigma(C)), C = H W a1 1^T + 1 (H W a2)^T; Z = Psi H W."""
    n = len(rp) - 1
    A = dense_mask(rp, ci, n)
    Ht, Wt, at = _t(H, True), _t(W, True), _t(a, True)
    kout = Wt.shape[1]
    d = kout // heads
    P = Ht @ Wt
    Zs, Psis = [], []
    for h in range(heads):
        Ph = P[:, h * d:(h + 1) * d]
        s = Ph @ at[h, :d]
        t = Ph @ at[h, d:]
        C = s[:, None] + t[None, :]                       # virtual n x n (rank-1 structure)
        Psi = masked_softmax(torch.nn.functional.leaky_relu(C, slope), A)
        Psis.append(Psi)
        Zs.append(Psi @ Ph)
    Z = torch.cat(Zs, dim=1)
    Hout = act(Z, kind)
    out = {"Z": Z.detach().numpy(), "Hout": Hout.detach().numpy(),
           "Psi": [p.detach().numpy() for p in Psis]}
    if R is not None:
        (Hout * _t(R)).sum().backward()
        out.update(dH=Ht.grad.numpy(), dW=Wt.grad.numpy(), da=at.grad.numpy())
    return out


def agnn(rp, ci, H, W, R=None, beta=1.0, eps=1e-12, kind="relu"):
    """Psi = sm(beta A (.) (H_x (/) n n^T)); Z = (Psi H) W (aggregate first, :207)."""
    n = len(rp) - 1
    A = dense_mask(rp, ci, n)
    Ht, Wt = _t(H, True), _t(W, True)
    nu = torch.clamp(torch.linalg.norm(Ht, dim=1), min=eps)
    C = beta * (Ht @ Ht.T) / (nu[:, None] * nu[None, :])
    Psi = masked_softmax(C, A)
    X = Psi @ Ht
    Z = X @ Wt
    Hout = act(Z, kind)
    out = {"Z": Z.detach().numpy(), "Hout": Hout.detach().numpy(), "Psi": Psi.detach().numpy(),
           "X": X.detach().numpy()}
    if R is not None:
        (Hout * _t(R)).sum().backward()
        out.update(dH=Ht.grad.numpy(), dW=Wt.grad.numpy())
    return out


def va(rp, ci, H, W, R=None, kind="relu"):
    """PAPER.md:173 / Eq. 7 (:262): Psi = A (.) (H H^T); Z = Psi H W."""
    n = len(rp) - 1
    A = dense_mask(rp, ci, n).to(DT)
    Ht, Wt = _t(H, True), _t(W, True)
    Psi = A * (Ht @ Ht.T)
    X = Psi @ Ht
    Z = X @ Wt
    Hout = act(Z, kind)
    out = {"Z": Z.detach().numpy(), "Hout": Hout.detach().numpy(), "Psi": Psi.detach().numpy(),
           "X": X.detach().numpy()}
    if R is not None:
        (Hout * _t(R)).sum().backward()
        out.update(dH=Ht.grad.numpy(), dW=Wt.grad.numpy())
    return out


def va_closed_form(rp, ci, H, W, R, kind="relu"):
    """The paper's printed VA backward, Eq. 11-13, dense numpy.

    G = dL/dH_out (.) sigma'(Z); M = G W^T; N = A (.) (M H^T); N+ = N + N^T
    Gamma (= dL/dH) = N+ H + (A^T (.) H_x) M ; Y = H^T (A^T (.) H_x) G.
    """
    n = len(rp) - 1
    A = dense_mask(rp, ci, n).numpy().astype(np.float64)
    H = np.asarray(H, np.float64)
    W = np.asarray(W, np.float64)
    Hx = H @ H.T
    Z = (A * Hx) @ H @ W
    if kind == "relu":
        dsig = (Z > 0).astype(np.float64)
    elif kind == "elu":
        dsig = np.where(Z > 0, 1.0, np.exp(Z))
    else:
        dsig = np.ones_like(Z)
    G = np.asarray(R, np.float64) * dsig
    M = G @ W.T                       # Eq. 12
    N = A * (M @ H.T)                 # Eq. 12
    Gamma = (N + N.T) @ H + (A.T * Hx) @ M   # Eq. 11
    Y = H.T @ (A.T * Hx) @ G          # Eq. 13
    return {"dH": Gamma, "dW": Y, "Z": Z}
