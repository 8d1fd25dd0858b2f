"""Seeded synthetic inputs (graphs, features, weights, upstream gradients).

Shared by both sides of every parity check: the oracle side calls the host
functions, the GPU path calls the device kernels; both evaluate the same
counter-based RNG in ``agnn_gen.h`` and are bit-identical.  This module holds
none of the A-GNN arithmetic (no projection, scoring, softmax or aggregation).

Workload recipes follow BASELINE.json ``configs`` and SURVEY.md §8(d); the
paper's own graphs are Graph500-style Kronecker and
uniform random "Rand" graphs.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os

import numpy as np

from .. import _build

ER, KRON, RMAT = 0, 1, 2
KIND = {"er": ER, "kron": KRON, "rmat": RMAT}
STREAM_GRAPH, STREAM_H, STREAM_R = 0, 1, 200


def STREAM_W(layer: int) -> int:
    return 2 + layer


def STREAM_A(layer: int) -> int:
    return 100 + layer


_lib = None


def lib():
    global _lib
    if _lib is None:
        so = _build.build_gen()
        _lib = ctypes.CDLL(so)
        for f in ("agen_edges_host", "agen_fill_host", "agen_fill_rows_host", "agen_edges_device",
                  "agen_fill_device"):
            getattr(_lib, f).restype = ctypes.c_int
    return _lib


def glorot_bound(k: int, kout: int) -> float:
    """sqrt(6/(k+k')) rounded to fp32 on the host, passed to both sides."""
    return float(np.sqrt(np.float32(6.0) / np.float32(k + kout), dtype=np.float32))


def edges(kind: int, seed: int, scale: int, n: int, n_samples: int):
    """Host edge samples (uint32 src, dst)."""
    src = np.empty(n_samples, dtype=np.uint32)
    dst = np.empty(n_samples, dtype=np.uint32)
    lib().agen_edges_host(ctypes.c_int(kind), ctypes.c_uint64(seed), ctypes.c_int(scale),
                          ctypes.c_uint64(n), ctypes.c_uint64(n_samples),
                          src.ctypes.data_as(ctypes.c_void_p), dst.ctypes.data_as(ctypes.c_void_p))
    return src, dst


def fill(seed: int, stream: int, shape, scale: float = 1.0, offset: int = 0) -> np.ndarray:
    """Host fp32 tensor of U[-1,1) * scale draws."""
    out = np.empty(shape, dtype=np.float32)
    lib().agen_fill_host(ctypes.c_uint64(seed), ctypes.c_uint64(stream), ctypes.c_uint64(offset),
                         ctypes.c_uint64(out.size), ctypes.c_float(scale),
                         out.ctypes.data_as(ctypes.c_void_p))
    return out


def fill_rows(seed: int, stream: int, ids, width: int, scale: float = 1.0) -> np.ndarray:
    """Host rows `ids` of a [*, width] fill() tensor (same values, without the rest)."""
    ids = np.ascontiguousarray(ids, dtype=np.int64)
    out = np.empty((len(ids), width), dtype=np.float32)
    lib().agen_fill_rows_host(ctypes.c_uint64(seed), ctypes.c_uint64(stream),
                              ids.ctypes.data_as(ctypes.c_void_p), ctypes.c_int64(len(ids)),
                              ctypes.c_int64(width), ctypes.c_float(scale),
                              out.ctypes.data_as(ctypes.c_void_p))
    return out


def edges_device(kind, seed, scale, n, n_samples, src_ptr: int, dst_ptr: int, stream: int = 0):
    rc = lib().agen_edges_device(ctypes.c_int(kind), ctypes.c_uint64(seed), ctypes.c_int(scale),
                                 ctypes.c_uint64(n), ctypes.c_uint64(n_samples),
                                 ctypes.c_void_p(src_ptr), ctypes.c_void_p(dst_ptr),
                                 ctypes.c_void_p(stream))
    if rc:
        raise RuntimeError("agen_edges_device failed")


def fill_device(seed, stream_id, count, scale, out_ptr: int, stream: int = 0, offset: int = 0):
    rc = lib().agen_fill_device(ctypes.c_uint64(seed), ctypes.c_uint64(stream_id),
                                ctypes.c_uint64(offset), ctypes.c_uint64(count),
                                ctypes.c_float(scale), ctypes.c_void_p(out_ptr),
                                ctypes.c_void_p(stream))
    if rc:
        raise RuntimeError("agen_fill_device failed")


@dataclasses.dataclass(frozen=True)
class Workload:
    """One BASELINE.json config as a concrete synthetic input recipe."""
    name: str
    model: str            # "gat" | "agnn" | "va" | "cgnn"
    graph: str            # "er" | "kron" | "rmat"
    scale: int            # log2 n (ER: n need not be a power of two)
    n: int
    n_samples: int        # undirected edge samples before preprocessing
    k: int                # features in = features out (k = k')
    heads: int
    layers: int
    seed: int = 1
    act: str = "relu"
    slope: float = 0.2
    beta: float = 1.0
    eps: float = 1e-12
    train: bool = False   # step = fwd + bwd + SGD update (C4) instead of fwd + bwd
    agg: str = "sum"      # C-GNN aggregation semiring (model "cgnn")
    lr: float = 1e-3
    prec: str = "fp32"    # "bf16": GAT P and G stored as bfloat16 (include/agnn.h AGNN_PREC_BF16)

    @property
    def kind(self) -> int:
        return KIND[self.graph]

    def weight_shapes(self, layer: int):
        d = self.k // self.heads
        return (self.k, self.k), ((self.heads, 2 * d) if self.model == "gat" else None)

    def host_inputs(self):
        """H, [W^l], [a^l], R on the host (fp32)."""
        H = fill(self.seed, STREAM_H, (self.n, self.k))
        bound = glorot_bound(self.k, self.k)
        Ws, As = [], []
        for l in range(self.layers):
            wshape, ashape = self.weight_shapes(l)
            Ws.append(fill(self.seed, STREAM_W(l), wshape, bound))
            As.append(fill(self.seed, STREAM_A(l), ashape, bound) if ashape else None)
        R = fill(self.seed, STREAM_R, (self.n, self.k))
        return H, Ws, As, R

    def host_edges(self):
        return edges(self.kind, self.seed, self.scale, self.n, self.n_samples)


def _kron(name, model, scale, ef, k, heads, layers, graph="kron", **kw):
    return Workload(name, model, graph, scale, 1 << scale, ef << scale, k, heads, layers, **kw)


# BASELINE.json configs[0..4]
CONFIGS = {
    "C1": Workload("C1", "gat", "er", 10, 1024, 7680, 16, 1, 1),
    "C2": _kron("C2", "gat", 16, 8, 64, 1, 2),
    "C3": _kron("C3", "agnn", 20, 16, 128, 1, 3, graph="rmat"),
    "C4": _kron("C4", "va", 22, 32, 256, 1, 1, train=True),   # "training step (fwd+bwd+SGD)"
    "C5": _kron("C5", "gat", 24, 32, 128, 4, 1),
}


def describe(w: Workload) -> str:
    return (f"{w.model.upper()} {w.layers} layer(s), {w.graph} n=2^{w.scale} samples={w.n_samples}, "
            f"k={w.k}, heads={w.heads}, seed={w.seed}")


__all__ = ["edges", "fill", "edges_device", "fill_device", "glorot_bound", "Workload", "CONFIGS",
           "ER", "KRON", "RMAT", "STREAM_H", "STREAM_R", "STREAM_W", "STREAM_A", "lib", "describe"]

_ = os  # keep import for future path helpers
