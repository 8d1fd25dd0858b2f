"""ORACLE — ctypes wrapper around oracle/liboracle.so (FP64, plain C).

TEST INFRASTRUCTURE ONLY: imported by tests/, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs, never by the
product package.  See agnn_oracle.c for the paper passages each routine
transcribes.  All arrays are numpy; floating inputs are converted to float64.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "agnn_oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

ACT = {"none": 0, "relu": 1, "elu": 2}
CSR_SYMMETRIZE, CSR_SELF_LOOPS, CSR_CONNECT_ISOLATED = 1, 2, 4


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain -O2, OpenMP over rows)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               _SRC, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_SO)
        _lib.oracle_csr_capacity.restype = ctypes.c_int64
    return _lib


def _p(x):
    return x.ctypes.data_as(ctypes.c_void_p)


def _d(x):
    return np.ascontiguousarray(x, dtype=np.float64)


def _i64(v):
    return ctypes.c_int64(int(v))


def csr_build(n, src, dst, flags=CSR_SYMMETRIZE | CSR_SELF_LOOPS | CSR_CONNECT_ISOLATED):
    """Canonical CSR (readings A1-A3, A21) from edge samples."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    L = lib()
    cap = L.oracle_csr_capacity(_i64(n), _i64(len(src)))
    rp = np.zeros(n + 1, dtype=np.int64)
    ci = np.zeros(max(cap, 1), dtype=np.int32)
    nnz = ctypes.c_int64(0)
    rc = L.oracle_csr_build(_i64(n), _p(src), _p(dst), _i64(len(src)), ctypes.c_uint32(flags),
                            _p(rp), _p(ci), ctypes.byref(nnz))
    if rc:
        raise ValueError(f"oracle_csr_build failed ({rc})")
    return rp, ci[: nnz.value].copy()


def partition(rp, world, c_v=4):
    """1D row-block bounds (reading A20)."""
    rp = np.ascontiguousarray(rp, dtype=np.int64)
    b = np.zeros(world + 1, dtype=np.int64)
    rc = lib().oracle_partition(_i64(len(rp) - 1), _p(rp), ctypes.c_int(world), _i64(c_v), _p(b))
    if rc:
        raise ValueError("oracle_partition failed")
    return b


def _csr(rp, ci):
    return (np.ascontiguousarray(rp, dtype=np.int64), np.ascontiguousarray(ci, dtype=np.int32),
            len(rp) - 1, int(rp[-1]))


def gat_forward(rp, ci, H, W, a, heads, slope=0.2, act="relu", bf16=False):
    """bf16: BF16 storage mode (P stored as bf16; out["P"] is the stored P~)."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W, a = _d(H), _d(W), _d(a)
    k, kout = W.shape
    out = {x: np.zeros((n, kout)) for x in ("P", "Z", "Hout")}
    out.update({x: np.zeros((n, heads)) for x in ("s", "t", "m", "l")})
    out["alpha"] = np.zeros((nnz, heads))
    fn = lib().oracle_gat_forward_bf16 if bf16 else lib().oracle_gat_forward
    rc = fn(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), ctypes.c_int(heads),
        _p(H), _p(W), _p(a), ctypes.c_double(slope), ctypes.c_int(ACT[act]),
        _p(out["P"]), _p(out["s"]), _p(out["t"]), _p(out["alpha"]), _p(out["m"]), _p(out["l"]),
        _p(out["Z"]), _p(out["Hout"]))
    if rc:
        raise ValueError("oracle_gat_forward failed")
    return out


def gat_backward(rp, ci, H, W, a, heads, fwd, dHout, slope=0.2, act="relu", bf16=False):
    """bf16: BF16 storage mode (G stored as bf16; fwd from gat_forward(bf16=True))."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W, a, dHout = _d(H), _d(W), _d(a), _d(dHout)
    k, kout = W.shape
    d = kout // heads
    out = {"dH": np.zeros((n, k)), "dW": np.zeros((k, kout)), "da": np.zeros((heads, 2 * d)),
           "G": np.zeros((n, kout)), "dP": np.zeros((n, kout))}
    fn = lib().oracle_gat_backward_bf16 if bf16 else lib().oracle_gat_backward
    rc = fn(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), ctypes.c_int(heads),
        _p(H), _p(W), _p(a), ctypes.c_double(slope), ctypes.c_int(ACT[act]),
        _p(fwd["P"]), _p(fwd["s"]), _p(fwd["t"]), _p(fwd["alpha"]), _p(fwd["Z"]), _p(dHout),
        _p(out["dH"]), _p(out["dW"]), _p(out["da"]), _p(out["G"]), _p(out["dP"]))
    if rc:
        raise ValueError("oracle_gat_backward failed")
    return out


def bf16_round(x):
    """round(fp32(x)) to the nearest bfloat16 (ties to even), in the oracle's C."""
    y = np.array(x, dtype=np.float64, copy=True, order="C")
    lib().oracle_bf16_round(_i64(y.size), _p(y))
    return y


def agnn_forward(rp, ci, H, W, beta=1.0, eps=1e-12, act="relu", bf16=False):
    """bf16: BF16 storage mode (reading B2): the layer computes on H~ = bf16(H)."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W = (bf16_round(H) if bf16 else _d(H)), _d(W)
    k, kout = W.shape
    out = {"nu": np.zeros(n), "alpha": np.zeros(nnz), "m": np.zeros(n), "l": np.zeros(n),
           "X": np.zeros((n, k)), "Z": np.zeros((n, kout)), "Hout": np.zeros((n, kout))}
    rc = lib().oracle_agnn_forward(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_double(beta), ctypes.c_double(eps), ctypes.c_int(ACT[act]),
        _p(out["nu"]), _p(out["alpha"]), _p(out["m"]), _p(out["l"]), _p(out["X"]), _p(out["Z"]),
        _p(out["Hout"]))
    if rc:
        raise ValueError("oracle_agnn_forward failed")
    return out


def agnn_backward(rp, ci, H, W, fwd, dHout, beta=1.0, eps=1e-12, act="relu", bf16=False):
    """bf16: BF16 storage mode (reading B2): H~ = bf16(H) and M~ = bf16(G W^T)."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W, dHout = (bf16_round(H) if bf16 else _d(H)), _d(W), _d(dHout)
    k, kout = W.shape
    out = {"dH": np.zeros((n, k)), "dW": np.zeros((k, kout))}
    fn = lib().oracle_agnn_backward_bf16 if bf16 else lib().oracle_agnn_backward
    rc = fn(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_double(beta), ctypes.c_double(eps), ctypes.c_int(ACT[act]),
        _p(fwd["nu"]), _p(fwd["alpha"]), _p(fwd["X"]), _p(fwd["Z"]), _p(dHout),
        _p(out["dH"]), _p(out["dW"]))
    if rc:
        raise ValueError("oracle_agnn_backward failed")
    return out


def va_forward(rp, ci, H, W, act="relu", bf16=False):
    """bf16: BF16 storage mode (reading B2): the layer computes on H~ = bf16(H)."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W = (bf16_round(H) if bf16 else _d(H)), _d(W)
    k, kout = W.shape
    out = {"S": np.zeros(nnz), "X": np.zeros((n, k)), "Z": np.zeros((n, kout)),
           "Hout": np.zeros((n, kout))}
    rc = lib().oracle_va_forward(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_int(ACT[act]), _p(out["S"]), _p(out["X"]), _p(out["Z"]), _p(out["Hout"]))
    if rc:
        raise ValueError("oracle_va_forward failed")
    return out


def va_backward(rp, ci, H, W, fwd, dHout, act="relu", bf16=False):
    """bf16: BF16 storage mode (reading B2): H~ = bf16(H) and M~ = bf16(G W^T)."""
    rp, ci, n, nnz = _csr(rp, ci)
    H, W, dHout = (bf16_round(H) if bf16 else _d(H)), _d(W), _d(dHout)
    k, kout = W.shape
    out = {"dH": np.zeros((n, k)), "dW": np.zeros((k, kout))}
    fn = lib().oracle_va_backward_bf16 if bf16 else lib().oracle_va_backward
    rc = fn(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_int(ACT[act]), _p(fwd["S"]), _p(fwd["X"]), _p(fwd["Z"]), _p(dHout),
        _p(out["dH"]), _p(out["dW"]))
    if rc:
        raise ValueError("oracle_va_backward failed")
    return out


AGG = {"sum": 0, "mean": 1, "gcn": 2, "max": 3, "min": 4}


def cgnn_forward(rp, ci, H, W, agg="sum", act="relu"):
    rp, ci, n, nnz = _csr(rp, ci)
    H, W = _d(H), _d(W)
    k, kout = W.shape
    out = {"X": np.zeros((n, k)), "arg": np.full((n, k), -1, np.int32), "Z": np.zeros((n, kout)),
           "Hout": np.zeros((n, kout))}
    rc = lib().oracle_cgnn_forward(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_int(AGG[agg]), ctypes.c_int(ACT[act]), _p(out["X"]), _p(out["arg"]),
        _p(out["Z"]), _p(out["Hout"]))
    if rc:
        raise ValueError("oracle_cgnn_forward failed")
    return out


def cgnn_backward(rp, ci, H, W, fwd, dHout, agg="sum", act="relu"):
    rp, ci, n, nnz = _csr(rp, ci)
    H, W, dHout = _d(H), _d(W), _d(dHout)
    k, kout = W.shape
    out = {"dH": np.zeros((n, k)), "dW": np.zeros((k, kout))}
    rc = lib().oracle_cgnn_backward(
        _i64(n), _p(rp), _p(ci), ctypes.c_int(k), ctypes.c_int(kout), _p(H), _p(W),
        ctypes.c_int(AGG[agg]), ctypes.c_int(ACT[act]), _p(fwd["X"]), _p(fwd["arg"]),
        _p(fwd["Z"]), _p(dHout), _p(out["dH"]), _p(out["dW"]))
    if rc:
        raise ValueError("oracle_cgnn_backward failed")
    return out


def layer(model, rp, ci, H, W, a=None, heads=1, dHout=None, act="relu", slope=0.2, beta=1.0,
          eps=1e-12, agg="sum", bf16=False):
    """Forward (+ backward when dHout is given) of one layer of `model`."""
    if model == "gat":
        f = gat_forward(rp, ci, H, W, a, heads, slope, act, bf16)
        b = (gat_backward(rp, ci, H, W, a, heads, f, dHout, slope, act, bf16)
             if dHout is not None else None)
    elif model == "agnn":
        f = agnn_forward(rp, ci, H, W, beta, eps, act, bf16)
        b = (agnn_backward(rp, ci, H, W, f, dHout, beta, eps, act, bf16)
             if dHout is not None else None)
    elif model == "va":
        f = va_forward(rp, ci, H, W, act, bf16)
        b = va_backward(rp, ci, H, W, f, dHout, act, bf16) if dHout is not None else None
    elif model == "cgnn":
        f = cgnn_forward(rp, ci, H, W, agg, act)
        b = cgnn_backward(rp, ci, H, W, f, dHout, agg, act) if dHout is not None else None
    else:
        raise ValueError(model)
    return f, b
