"""Thin Python binding of libagnn.so (include/agnn.h) — argument marshalling only.

Every step of the layer runs in the library's CUDA kernels; this module only
turns torch tensors into device pointers and streams into handles.  There is
no CPU or PyTorch fallback: if libagnn.so is missing or no CUDA device is
present, the calls raise.  The names mirror the C ABI (agnn_plan / agnn_forward
/ agnn_backward, Eq. 1 and :250-254 Eq. 6).
"""
from __future__ import annotations

import ctypes
import os

from . import _build

VA, AGNN, GAT = 0, 1, 2
KIND = {"va": VA, "agnn": AGNN, "gat": GAT, "cgnn": 3}
AGG = {"sum": 0, "mean": 1, "gcn": 2, "max": 3, "min": 4}
ACT = {"none": 0, "relu": 1, "elu": 2}
PREC_FP32, PREC_TF32X3, PREC_BF16 = 0, 1, 2
PREC = {"fp32": PREC_FP32, "tf32x3": PREC_TF32X3, "bf16": PREC_BF16}
CSR_SYMMETRIC, PLAN_VERIFY_SYMMETRY = 1, 2
BUILD_SYMMETRIZE, BUILD_SELF_LOOPS, BUILD_CONNECT_ISOLATED = 1, 2, 4
BUILD_PAPER = BUILD_SYMMETRIZE | BUILD_SELF_LOOPS | BUILD_CONNECT_ISOLATED

STATUS = {0: "AGNN_OK", 1: "AGNN_EINVAL", 2: "AGNN_ECUDA", 3: "AGNN_ENCCL", 4: "AGNN_ENOMEM",
          5: "AGNN_EUNSUPPORTED", 6: "AGNN_ESTATE"}

# every symbol include/agnn.h declares (tests check the .so exports all of them)
EXPORTS = ("agnn_partition", "agnn_plan_create", "agnn_plan_create_ex", "agnn_plan_destroy", "agnn_plan_info",
           "agnn_plan_csc", "agnn_loss_inner", "agnn_sgd_step",
           "agnn_ipc_export", "agnn_plan_ctl_export", "agnn_plan_connect", "agnn_plan_register",
           "agnn_model_create", "agnn_model_destroy", "agnn_saved_bytes", "agnn_workspace_bytes",
           "agnn_forward", "agnn_backward", "agnn_debug_attention", "agnn_debug_gemm",
           "agnn_debug_gemm_tn", "agnn_debug_gemm_tn_ws_bytes",
           "agnn_launch_count",
           "agnn_profile_enable", "agnn_profile_report", "agnn_profile_reset",
           "agnn_nccl_unique_id", "agnn_csr_build", "agnn_free", "agnn_status_string",
           "agnn_last_error")


class AgnnError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class CSR(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p),
                ("flags", ctypes.c_uint32)]


class PlanOptions(ctypes.Structure):
    """agnn_plan_options (include/agnn.h); a field < 0 (0 for chunk_edges) = default."""
    _fields_ = [("chunk_edges", ctypes.c_int32), ("short_edges", ctypes.c_int32),
                ("short_bundles", ctypes.c_int32), ("gat_factored", ctypes.c_int32),
                ("l2_hot_mb", ctypes.c_int32), ("spmmm", ctypes.c_int32)]

    @classmethod
    def make(cls, chunk_edges=0, short_edges=-1, short_bundles=-1, gat_factored=-1, l2_hot_mb=-1,
             spmmm=-1):
        return cls(chunk_edges, short_edges, short_bundles, gat_factored, l2_hot_mb, spmmm)


class Dist(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int), ("world", ctypes.c_int),
                ("nccl_unique_id", ctypes.c_void_p), ("bounds", ctypes.c_void_p)]


class LayerDesc(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("k_in", ctypes.c_int), ("k_out", ctypes.c_int),
                ("heads", ctypes.c_int), ("act", ctypes.c_int), ("prec", ctypes.c_int),
                ("negative_slope", ctypes.c_float), ("beta", ctypes.c_float),
                ("eps", ctypes.c_float), ("agg", ctypes.c_int)]


_lib = None


def lib(build: bool = True):
    """Load libagnn.so (building it in-tree if stale).  Raises if unavailable."""
    global _lib
    if _lib is None:
        # AGNN_LIB: an explicit libagnn.so (e.g. a build of another revision for A/B timing)
        so = os.environ.get("AGNN_LIB") or (_build.build_agnn() if build else _build.AGNN_SO)
        if not os.path.exists(so):
            raise RuntimeError(f"libagnn.so not found at {so}; run __graft_entry__.build()")
        L = ctypes.CDLL(so)
        L.agnn_status_string.restype = ctypes.c_char_p
        L.agnn_last_error.restype = ctypes.c_char_p
        L.agnn_launch_count.restype = ctypes.c_uint64
        L.agnn_debug_gemm_tn_ws_bytes.restype = ctypes.c_size_t
        for name in EXPORTS:
            fn = getattr(L, name)
            if name not in ("agnn_status_string", "agnn_last_error", "agnn_launch_count",
                            "agnn_free", "agnn_debug_gemm_tn_ws_bytes"):
                fn.restype = ctypes.c_int
        _lib = L
    return _lib


def _check(rc):
    if rc != 0:
        raise AgnnError(rc, lib().agnn_last_error().decode(errors="replace"))


def _ptr(t):
    return ctypes.c_void_p(0 if t is None else t.data_ptr())


def _stream(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


def launch_count() -> int:
    return int(lib().agnn_launch_count())


def profile_enable(on: bool = True):
    _check(lib().agnn_profile_enable(ctypes.c_int(1 if on else 0)))


def profile_reset():
    _check(lib().agnn_profile_reset())


def profile_report() -> dict:
    """{kernel name: (launches, total_ms)} accumulated since the last reset (synchronises)."""
    buf = ctypes.create_string_buffer(1 << 16)
    _check(lib().agnn_profile_report(buf, ctypes.c_size_t(len(buf))))
    out = {}
    for line in buf.value.decode().splitlines():
        name, cnt, ms = line.rsplit(" ", 2)
        out[name] = (int(cnt), float(ms))
    return out


def ipc_export(tensor):
    """(64-byte CUDA IPC handle of the allocation holding `tensor`, byte offset)."""
    h = ctypes.create_string_buffer(64)
    off = ctypes.c_int64()
    _check(lib().agnn_ipc_export(ctypes.c_void_p(tensor.data_ptr()), h, ctypes.byref(off)))
    return h.raw, off.value


LOSS_SCRATCH = 1024  # AGNN_LOSS_SCRATCH


def loss_inner(R, H, scratch, loss, stream=None):
    """agnn_loss_inner: loss[0] = <R, H> in fp64 (device); scratch: >= LOSS_SCRATCH doubles."""
    assert R.numel() == H.numel() and scratch.numel() >= LOSS_SCRATCH
    _check(lib().agnn_loss_inner(_ptr(R), _ptr(H), ctypes.c_int64(R.numel()), _ptr(scratch),
                                 _ptr(loss), _stream(stream)))


def sgd_step(W, dW, lr, stream=None):
    """agnn_sgd_step: W -= lr * dW on the device."""
    assert W.numel() == dW.numel()
    _check(lib().agnn_sgd_step(_ptr(W), _ptr(dW), ctypes.c_int64(W.numel()), ctypes.c_float(lr),
                               _stream(stream)))


def debug_gemm(A, B, C, stream=None):
    """C = A @ B.T through the library's projection GEMM (test-only)."""
    _check(lib().agnn_debug_gemm(_ptr(A), ctypes.c_int64(A.shape[0]), ctypes.c_int(A.shape[1]),
                                 _ptr(B), ctypes.c_int(B.shape[0]), _ptr(C), _stream(stream)))


def debug_gemm_tn(A, B, C, stream=None):
    """C = A.T @ B through the library's weight-gradient GEMM (test-only)."""
    import torch
    nbytes = lib().agnn_debug_gemm_tn_ws_bytes(ctypes.c_int(A.shape[1]), ctypes.c_int(B.shape[1]))
    ws = torch.empty(nbytes // 4 + 1, dtype=torch.float32, device=A.device)
    _check(lib().agnn_debug_gemm_tn(_ptr(A), ctypes.c_int64(A.shape[0]), ctypes.c_int(A.shape[1]),
                                    _ptr(B), ctypes.c_int(B.shape[1]), _ptr(C), _ptr(ws),
                                    _stream(stream)))


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().agnn_nccl_unique_id(buf))
    return buf.raw


def partition(row_ptr_host, world: int, c_v: int = 4):
    """agnn_partition on a host int64 row_ptr (numpy); returns numpy bounds[world+1]."""
    import numpy as np
    rp = np.ascontiguousarray(row_ptr_host, dtype=np.int64)
    b = np.zeros(world + 1, dtype=np.int64)
    _check(lib().agnn_partition(ctypes.c_int64(len(rp) - 1), rp.ctypes.data_as(ctypes.c_void_p),
                                ctypes.c_int(world), ctypes.c_int64(c_v),
                                b.ctypes.data_as(ctypes.c_void_p)))
    return b


class _DeviceArray:
    """Library-allocated device buffer exposed to torch via __cuda_array_interface__."""

    def __init__(self, ptr, n, typestr):
        self.ptr, self.n = ptr, n
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr,
                                         "data": (ptr, False), "version": 3, "strides": None}

    def __del__(self):
        if self.ptr and _lib is not None:
            _lib.agnn_free(ctypes.c_void_p(self.ptr))
            self.ptr = 0


def csr_build(n: int, src, dst, flags: int = BUILD_PAPER, stream=None):
    """agnn_csr_build on device uint32 edge samples -> (row_ptr int64[n+1], col_idx int32)."""
    import torch
    row_ptr = torch.empty(n + 1, dtype=torch.int64, device=src.device)
    col = ctypes.c_void_p(0)
    nnz = ctypes.c_int64(0)
    _check(lib().agnn_csr_build(ctypes.c_int64(n), _ptr(src), _ptr(dst), ctypes.c_int64(src.numel()),
                                ctypes.c_uint32(flags), _ptr(row_ptr), ctypes.byref(col),
                                ctypes.byref(nnz), _stream(stream)))
    holder = _DeviceArray(col.value or 0, nnz.value, "<i4")
    col_t = torch.as_tensor(holder, device=src.device) if nnz.value > 0 else \
        torch.empty(0, dtype=torch.int32, device=src.device)
    col_t._agnn_holder = holder  # keep the allocation alive with the tensor
    return row_ptr, col_t


class Plan:
    """agnn_plan_create: validated CSR + work lists (+ NCCL communicator when world > 1)."""

    def __init__(self, row_ptr, col_idx, n, row_begin=0, row_end=None, symmetric=True,
                 rank=0, world=1, nccl_unique_id: bytes | None = None, bounds=None, stream=None,
                 options: dict | None = None, verify_symmetry: bool = False):
        self.row_ptr, self.col_idx = row_ptr, col_idx  # keep the caller's CSR alive
        row_end = n if row_end is None else row_end
        flags = (CSR_SYMMETRIC if symmetric else 0) | (PLAN_VERIFY_SYMMETRY if verify_symmetry else 0)
        self._csr = CSR(n, row_begin, row_end, row_ptr.data_ptr(), col_idx.data_ptr(), flags)
        self._opts = PlanOptions.make(**(options or {}))
        dist = None
        if world > 1:
            import numpy as np
            self._bounds = np.ascontiguousarray(bounds, dtype=np.int64)
            uid = None
            if nccl_unique_id is not None:  # NCCL exchange; None: peer-memory exchange
                self._uid = ctypes.create_string_buffer(bytes(nccl_unique_id), 128)
                uid = ctypes.cast(self._uid, ctypes.c_void_p)
            dist = Dist(rank, world, uid, self._bounds.ctypes.data_as(ctypes.c_void_p))
        h = ctypes.c_void_p()
        _check(lib().agnn_plan_create_ex(ctypes.byref(self._csr),
                                         ctypes.byref(dist) if dist is not None else None,
                                         ctypes.byref(self._opts), _stream(stream), ctypes.byref(h)))
        self.handle = h
        self.n, self.row_begin, self.row_end = n, row_begin, row_end
        self.n_local = row_end - row_begin

    def info(self) -> dict:
        a = (ctypes.c_int64 * 12)()
        _check(lib().agnn_plan_info(self.handle, a))
        keys = ("n_local", "nnz", "light_rows", "heavy_rows", "heavy_chunks", "chunk", "max_degree",
                "n", "short_rows", "short_max", "recv_rows", "send_rows")
        return dict(zip(keys, list(a)))

    # ---- peer-memory exchange setup (world > 1 without an NCCL id) -------------
    def ctl_export(self):
        """(handle bytes, offset) of this rank's control block."""
        h = ctypes.create_string_buffer(64)
        off = ctypes.c_int64()
        _check(lib().agnn_plan_ctl_export(self.handle, h, ctypes.byref(off)))
        return h.raw, off.value

    def connect(self, exports):
        """exports: [(handle, offset)] of every rank's control block, rank order."""
        hs = b"".join(h for h, _ in exports)
        offs = (ctypes.c_int64 * len(exports))(*[o for _, o in exports])
        _check(lib().agnn_plan_connect(self.handle, hs, offs))

    def register(self, tensor, exports):
        """Map every rank's copy of `tensor` (its replicated prefix sits at the same offsets)."""
        hs = b"".join(h for h, _ in exports)
        offs = (ctypes.c_int64 * len(exports))(*[o for _, o in exports])
        _check(lib().agnn_plan_register(self.handle, ctypes.c_void_p(tensor.data_ptr()),
                                        ctypes.c_size_t(tensor.numel() * tensor.element_size()),
                                        hs, offs))

    def csc(self, perm=True, stream=None):
        """agnn_plan_csc: (col_ptr int64 [n+1], row_idx int32 [nnz], perm int64 [nnz] | None)."""
        import torch
        dev = self.row_ptr.device
        nnz = int(self.col_idx.numel())
        cp = torch.empty(self.n + 1, dtype=torch.int64, device=dev)
        ri = torch.empty(max(nnz, 1), dtype=torch.int32, device=dev)
        pm = torch.empty(max(nnz, 1), dtype=torch.int64, device=dev) if perm else None
        _check(lib().agnn_plan_csc(self.handle, _ptr(cp), _ptr(ri),
                                   _ptr(pm) if pm is not None else None, _stream(stream)))
        return cp, ri[:nnz], (pm[:nnz] if pm is not None else None)

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:
            _lib.agnn_plan_destroy(self.handle)
            self.handle = None


def layer_desc(kind, k_in, k_out, heads=1, act="relu", prec=PREC_FP32, negative_slope=0.2,
               beta=1.0, eps=1e-12, agg="sum") -> LayerDesc:
    return LayerDesc(KIND[kind] if isinstance(kind, str) else kind, k_in, k_out, heads,
                     ACT[act] if isinstance(act, str) else act, prec, negative_slope, beta, eps,
                     AGG[agg] if isinstance(agg, str) else agg)


class Model:
    """agnn_model_create over a plan; forward/backward are the C entry points."""

    def __init__(self, plan: Plan, descs):
        self.plan = plan
        self.descs = list(descs)
        arr = (LayerDesc * len(self.descs))(*self.descs)
        h = ctypes.c_void_p()
        _check(lib().agnn_model_create(plan.handle, len(self.descs), arr, ctypes.byref(h)))
        self.handle = h

    def saved_bytes(self, layer: int) -> int:
        b = ctypes.c_size_t(0)
        _check(lib().agnn_saved_bytes(self.handle, layer, ctypes.byref(b)))
        return b.value

    def workspace_bytes(self, layer: int) -> int:
        b = ctypes.c_size_t(0)
        _check(lib().agnn_workspace_bytes(self.handle, layer, ctypes.byref(b)))
        return b.value

    def forward(self, layer, W, a, H_in, H_out, saved, workspace, stream=None):
        _check(lib().agnn_forward(self.handle, layer, _ptr(W), _ptr(a), _ptr(H_in), _ptr(H_out),
                                  _ptr(saved), _ptr(workspace), _stream(stream)))

    def backward(self, layer, W, a, H_in, saved, dH_out, dH_in, dW, da, workspace, stream=None):
        _check(lib().agnn_backward(self.handle, layer, _ptr(W), _ptr(a), _ptr(H_in), _ptr(saved),
                                   _ptr(dH_out), _ptr(dH_in), _ptr(dW), _ptr(da), _ptr(workspace),
                                   _stream(stream)))

    def debug_attention(self, layer, saved, H_in, edge_pos, out, stream=None):
        _check(lib().agnn_debug_attention(self.handle, layer, _ptr(saved), _ptr(H_in),
                                          _ptr(edge_pos), ctypes.c_int64(edge_pos.numel()),
                                          _ptr(out), _stream(stream)))

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:
            _lib.agnn_model_destroy(self.handle)
            self.handle = None
