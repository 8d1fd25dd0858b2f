"""World-size-2 checks of the N > 1 host path on CPU (gloo, 127.0.0.1).

The NCCL exchange itself needs several GPUs; what runs here is everything
around it: the 1D row-block partition each rank derives independently
(agnn_partition, reading A20), the CSR slicing of runner.row_block, the
all-gather-v semantics the library implements with grouped broadcasts (row
blocks of different sizes re-assembled in global row order), the NCCL unique-id
broadcast and the max-over-ranks timing reduction bench.py uses.
"""
from __future__ import annotations

import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    try:
        sys.path.insert(0, ROOT)
        sys.path.insert(0, os.path.join(ROOT, "oracle"))
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        from paper_conf_sc_bestarglzcgssci23_b200 import gen, runner
        w = gen.Workload("g", "gat", "rmat", 11, 2048, 16 * 2048, 16, 2, 1)  # skewed R-MAT
        src, dst = w.host_edges()
        rp, ci = oracle.csr_build(w.n, src, dst)
        bounds, b0, b1, e0, e1 = runner.row_block(rp, world, rank)
        # every rank derives the same bounds, bit-exact with the oracle's formula
        assert np.array_equal(bounds, oracle.partition(rp, world, 4))
        allb = [None] * world
        dist.all_gather_object(allb, bounds.tolist())
        assert all(b == bounds.tolist() for b in allb)
        # local CSR slice is a valid CSR of the rank's rows with global column ids
        lrp = rp[b0:b1 + 1] - e0
        lci = ci[e0:e1]
        assert lrp[0] == 0 and lrp[-1] == len(lci)
        # all-gather-v of row blocks (what allgather_rows does with grouped ncclBroadcast)
        H, Ws, As, R = w.host_inputs()
        P_local = torch.from_numpy(H[b0:b1] @ Ws[0])
        blocks = [torch.zeros((int(bounds[r + 1] - bounds[r]), P_local.shape[1])) for r in range(world)]
        for r in range(world):
            buf = P_local.clone() if r == rank else blocks[r]
            dist.broadcast(buf, src=r)
            blocks[r] = buf
        P_full = torch.cat(blocks).numpy()
        assert np.allclose(P_full, H @ Ws[0], rtol=1e-6, atol=1e-6)
        # the oracle layer restricted to the rank's rows equals the full layer's rows
        f_full, _ = oracle.layer("gat", rp, ci, H, Ws[0], As[0], 2)
        sub_rp = np.concatenate([np.zeros(b0, np.int64), lrp + e0, np.full(w.n - b1, e1, np.int64)])
        sub_rp[:b0] = 0
        # rows outside the block are empty; columns stay global
        sub_ci = ci[e0:e1]
        sub_rp = np.concatenate([np.zeros(b0 + 1, np.int64), lrp[1:], np.full(w.n - b1, e1 - e0, np.int64)])
        f_loc, _ = oracle.layer("gat", sub_rp, sub_ci, H, Ws[0], As[0], 2)
        assert np.allclose(f_loc["Z"][b0:b1], f_full["Z"][b0:b1], rtol=1e-12, atol=1e-12)
        # unique-id broadcast + max-over-ranks timing, as bench.py does
        obj = [bytes(range(128)) if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        assert obj[0] == bytes(range(128))
        t = torch.tensor([float(rank + 1)])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        assert t.item() == world
        edges = torch.tensor([e1 - e0], dtype=torch.int64)
        dist.all_reduce(edges)
        assert edges.item() == len(ci)
        q.put((rank, "ok", b0, b1))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, "fail", traceback.format_exc(), None))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_rank_row_blocks_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    bad = [r for r in res if r[1] != "ok"]
    assert not bad, bad[0][2]
    spans = sorted((r[2], r[3]) for r in res)
    assert spans[0][0] == 0 and spans[-1][1] == 2048
    assert all(spans[i][1] == spans[i + 1][0] for i in range(len(spans) - 1))
