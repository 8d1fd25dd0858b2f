"""L-layer A-GNN training step over the C ABI (the "model" layer above the path).

PAPER.md:378: "a forward pass followed by backward pass, each with L layers";
PAPER.md:584 (GnnModel: forward/backward over GnnLayer).  This module only
allocates device memory with torch, generates the synthetic inputs with the
seeded generators, and calls agnn_forward / agnn_backward layer by layer; all
arithmetic runs in libagnn.so.  Multi-GPU: one process per GPU, 1D row blocks
(agnn_partition), NCCL inside the library; the process group only ships the
NCCL unique id.
"""
from __future__ import annotations

import dataclasses

import numpy as np
import torch

from . import agnn, gen


@dataclasses.dataclass
class Graph:
    n: int
    row_ptr: torch.Tensor      # full graph, device int64 [n+1]
    col_idx: torch.Tensor      # device int32 [nnz]
    nnz: int


def build_graph(w: gen.Workload, device, stream=None) -> Graph:
    """Generate the workload's edge samples on the device and build its canonical CSR."""
    src = torch.empty(w.n_samples, dtype=torch.int32, device=device)
    dst = torch.empty_like(src)
    s = (stream or torch.cuda.current_stream(device)).cuda_stream
    gen.edges_device(w.kind, w.seed, w.scale, w.n, w.n_samples, src.data_ptr(), dst.data_ptr(), s)
    rp, ci = agnn.csr_build(w.n, src, dst, agnn.BUILD_PAPER, stream=stream)
    del src, dst
    return Graph(w.n, rp, ci, int(ci.numel()))


def row_block(row_ptr_host, world: int, rank: int, c_v: int = 4):
    """1D row-block of `rank` (reading A20): (bounds, row_begin, row_end, edge_begin, edge_end).

    Pure host logic (agnn_partition from libagnn.so on the host row_ptr); the
    rank keeps rows [row_begin, row_end) and stored entries [edge_begin, edge_end)
    of the global CSR, with its local row_ptr = row_ptr[row_begin:row_end+1] - edge_begin.
    """
    rp = np.ascontiguousarray(row_ptr_host, dtype=np.int64)
    bounds = agnn.partition(rp, world, c_v) if world > 1 else np.array([0, len(rp) - 1], np.int64)
    b0, b1 = int(bounds[rank]), int(bounds[rank + 1])
    return bounds, b0, b1, int(rp[b0]), int(rp[b1])


class Stack:
    """Buffers + plan + model for one workload on this rank.

    world > 1: `nccl_uid` selects the NCCL exchange; without it the ranks exchange
    through peer memory, and `allgather_obj` (list <- object, every rank; e.g.
    torch.distributed.all_gather_object) moves the IPC handles at setup."""

    def __init__(self, w: gen.Workload, device="cuda", rank=0, world=1, nccl_uid=None,
                 c_v: int = 4, graph: Graph | None = None, inputs_on_device=True,
                 symmetric: bool = True, allgather_obj=None, plan_options: dict | None = None):
        self.w, self.device, self.rank, self.world = w, torch.device(device), rank, world
        self.stream = torch.cuda.current_stream(self.device)
        g = graph or build_graph(w, self.device)
        self.graph = g
        if world > 1:
            self.bounds, b0, b1, e0, e1 = row_block(g.row_ptr.cpu().numpy(), world, rank, c_v)
            self.row_ptr = (g.row_ptr[b0:b1 + 1] - e0).contiguous()
            self.col_idx = g.col_idx[e0:e1].contiguous()
        else:
            self.bounds = np.array([0, w.n], dtype=np.int64)
            b0, b1 = 0, w.n
            self.row_ptr, self.col_idx = g.row_ptr, g.col_idx
        self.row_begin, self.row_end, self.n_local = b0, b1, b1 - b0
        self.nnz_local = int(self.col_idx.numel())
        # symmetric=False: a directed pattern (reading A4); the plan builds its CSC
        self.plan = agnn.Plan(self.row_ptr, self.col_idx, w.n, b0, b1, symmetric=symmetric, rank=rank,
                              world=world, nccl_unique_id=nccl_uid, bounds=self.bounds,
                              options=plan_options)
        descs = [agnn.layer_desc(w.model, w.k, w.k, w.heads, w.act, prec=agnn.PREC[w.prec],
                                 negative_slope=w.slope,
                                 beta=w.beta, eps=w.eps, agg=w.agg) for _ in range(w.layers)]
        self.model = agnn.Model(self.plan, descs)
        self._alloc(inputs_on_device)
        if world > 1 and nccl_uid is None:
            if allgather_obj is None:
                import torch.distributed as dist

                def allgather_obj(obj):
                    out = [None] * world
                    dist.all_gather_object(out, obj)
                    return out
            self.plan.connect(allgather_obj(self.plan.ctl_export()))
            for t in self.saved + [self.ws]:   # same order and sizes on every rank
                self.plan.register(t, allgather_obj(agnn.ipc_export(t)))

    def _alloc(self, inputs_on_device):
        w, dev, nl = self.w, self.device, self.n_local
        f32 = dict(dtype=torch.float32, device=dev)
        s = self.stream.cuda_stream
        self.H = [torch.empty((nl, w.k), **f32) for _ in range(w.layers + 1)]   # H^0 .. H^L
        self.dH = [torch.empty((nl, w.k), **f32) for _ in range(w.layers + 1)]  # dL/dH^l
        bound = gen.glorot_bound(w.k, w.k)
        self.W, self.a, self.dW, self.da = [], [], [], []
        for l in range(w.layers):
            Wt = torch.empty((w.k, w.k), **f32)
            gen.fill_device(w.seed, gen.STREAM_W(l), Wt.numel(), bound, Wt.data_ptr(), s)
            self.W.append(Wt)
            self.dW.append(torch.empty_like(Wt))
            if w.model == "gat":
                at = torch.empty((w.heads, 2 * (w.k // w.heads)), **f32)
                gen.fill_device(w.seed, gen.STREAM_A(l), at.numel(), bound, at.data_ptr(), s)
                self.a.append(at)
                self.da.append(torch.empty_like(at))
            else:
                self.a.append(None)
                self.da.append(None)
        if inputs_on_device:
            gen.fill_device(w.seed, gen.STREAM_H, nl * w.k, 1.0, self.H[0].data_ptr(), s,
                            offset=self.row_begin * w.k)
            gen.fill_device(w.seed, gen.STREAM_R, nl * w.k, 1.0, self.dH[w.layers].data_ptr(), s,
                            offset=self.row_begin * w.k)
        self.saved = [torch.empty(self.model.saved_bytes(l), dtype=torch.uint8, device=dev)
                      for l in range(w.layers)]
        ws = max(self.model.workspace_bytes(l) for l in range(w.layers))
        self.ws = torch.empty(ws, dtype=torch.uint8, device=dev)

    def forward(self, inference=False):
        for l in range(self.w.layers):
            self.model.forward(l, self.W[l], self.a[l], self.H[l], self.H[l + 1],
                               None if inference else self.saved[l], self.ws, self.stream)

    def backward(self):
        for l in reversed(range(self.w.layers)):
            self.model.backward(l, self.W[l], self.a[l], self.H[l], self.saved[l], self.dH[l + 1],
                                self.dH[l], self.dW[l], self.da[l], self.ws, self.stream)

    def sgd(self, lr=None):
        """W^l -= lr dW^l (and a^l for GAT) on the device."""
        lr = self.w.lr if lr is None else lr
        for l in range(self.w.layers):
            agnn.sgd_step(self.W[l], self.dW[l], lr, self.stream)
            if self.a[l] is not None:
                agnn.sgd_step(self.a[l], self.da[l], lr, self.stream)

    def loss(self):
        """L = <R, H^L> (reading A13) into a device fp64 scalar (this rank's rows)."""
        if not hasattr(self, "_loss"):
            self._loss = torch.zeros(1, dtype=torch.float64, device=self.device)
            self._loss_ws = torch.empty(agnn.LOSS_SCRATCH, dtype=torch.float64, device=self.device)
        agnn.loss_inner(self.dH[self.w.layers], self.H[self.w.layers], self._loss_ws, self._loss,
                        self.stream)
        return self._loss

    def step(self):
        """One pass over all L layers (the bench 'step'): forward + backward, plus
        the SGD update for training workloads (C4: "training step (fwd+bwd+SGD)")."""
        self.forward()
        self.backward()
        if self.w.train:
            self.sgd()

    def edges_total(self) -> int:
        return self.graph.nnz
