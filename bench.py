#!/usr/bin/env python
"""bench.py — GAT/AGNN/VA layer fwd+bwd edges/s on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--impl ours|reference]

A "step" is one pass of the whole hot path over the synthetic workload: the
L-layer forward (projection GEMM, fused SDDMM -> edge softmax -> SpMM, sigma)
followed by the L-layer backward (prologue, fused recompute backward, weight-
gradient and dH GEMMs, and at N > 1 the NCCL exchanges).  edges/s = L * m / T
(m = nnz after preprocessing, global).

Default workload: C5 = GAT, 4 heads, k = 128, Kronecker n = 2^24 / ~1.0e9
edges, 1 layer — the north_star target (fits one B200).  Inputs (8.6 GB per
feature matrix) are far larger than the 126 MB L2, so no explicit flush.

Multi-GPU: one rank per GPU.  `--gpus N` with N > 1 outside torchrun re-launches
itself under torch.distributed.run (N processes); 1D row blocks; the all-gathers
of P / G are fused into the producing kernels as NVLink peer stores and dW, da
are all-reduced through peer memory (--comm peer, default; --comm nccl or
missing P2P access: NCCL inside libagnn.so); rank 0 prints the JSON line; time =
max over ranks of CUDA-event time.  Default scaling is strong (the named config
at every N); --weak grows the graph with N (n = 2^21 N, same edge factor,
S§8(d)).  AGNN_BENCH_SAME_GPU=1 (functional test only) runs every rank on cuda:0.

Roofline (S§8(d) "three numbers per sparse kernel"): `frac` = ncu-measured DRAM
bytes of the dominant pass per launch (profiles/ncu_traffic.json, stamped with
the hash of the kernel sources it was captured from; a stale entry is refused)
/ the live CUDA-event launch time / the measured HBM copy peak; `model_frac` =
the algorithmic byte model / time / peak (can exceed 1: L2 serves hub gathers);
`gather_peak_frac` = DRAM rate / the measured random-row gather rate.
"""
from __future__ import annotations

import argparse
import glob
import hashlib
import json
import os
import socket
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GAT layer fwd+bwd edges/s"
UNIT = "edges/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="C5")
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--comm", default="peer", choices=["peer", "nccl"],
                   help="multi-GPU exchange: peer memory (fused GEMM -> all-gather stores over "
                        "NVLink, flag barriers) or NCCL collectives")
    p.add_argument("--graph", default="auto", choices=["auto", "on", "off"],
                   help="time the step as one CUDA-graph replay (auto: small, launch-bound "
                        "workloads on one GPU)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-bf16-line", action="store_true",
                   help="skip the extra BF16-storage measurement of GAT k'=128 workloads")
    p.add_argument("--prec", default="fp32", choices=["fp32", "bf16"],
                   help="feature storage: fp32, or bf16 (GAT: P and G, AGNN/VA: H and M stored "
                        "as bfloat16, "
                        "fp32 arithmetic; include/agnn.h AGNN_PREC_BF16, reading B1)")
    p.add_argument("--scale", type=int, default=None,
                   help="override log2 n of the workload (same recipe and edge factor)")
    p.add_argument("--cpu-sample-scale", type=int, default=19,
                   help="log2 n of the bounded oracle sample (same recipe as the workload)")
    p.add_argument("--spmmm", type=int, default=-1, choices=[-1, 0, 1],
                   help="AGNN/VA k = 128 forward: 1 = fused SpMMM kernel (aggregation and "
                        "projection in one kernel, agnn_plan_options.spmmm), 0 = SpMM kernel + "
                        "tcgen05 GEMM, -1 = the library default")
    p.add_argument("--weak", action="store_true",
                   help="weak scaling: n = 2^21 x N vertices (same recipe and edge factor)")
    return p.parse_args()


# ----------------------------------------------------------------------------- launcher
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def maybe_relaunch(args):
    """--gpus N > 1 outside torchrun: run this script as N ranks under
    torch.distributed.run (one process per GPU) and exit with its status."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return
    if args.impl == "ours" and os.environ.get("AGNN_BENCH_SAME_GPU") != "1":
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            sys.exit(f"bench.py --gpus {args.gpus}: only {have} CUDA device(s) visible "
                     "(AGNN_BENCH_SAME_GPU=1 runs the ranks on one GPU as a functional test)")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
           "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


# ----------------------------------------------------------------------------- ncu stamps
# the practical HBM rate of random whole-row gathers of 512 B (scratch/gather_probe.cu,
# profiles/r01_gather_probe.txt: 24 warps / SM, 8 rows in flight): read-only gathers
# exceed the copy peak of MEASURED_PEAKS.json
GATHER_PEAK_GBS = 7272.0


def kernel_source_hash():
    """sha256 (first 16 hex) of the library sources the DRAM traffic was measured on."""
    h = hashlib.sha256()
    pkg = os.path.join(ROOT, "paper_conf_sc_bestarglzcgssci23_b200", "csrc")
    for f in sorted(glob.glob(os.path.join(pkg, "*.cu")) + glob.glob(os.path.join(pkg, "*.cuh")) +
                    glob.glob(os.path.join(ROOT, "include", "*.h"))):
        h.update(os.path.basename(f).encode())
        h.update(open(f, "rb").read())
    return h.hexdigest()[:16]


def ncu_traffic(key):
    """{kernel: DRAM bytes per launch} of workload `key`, or (None, why) when the
    committed capture is missing or was taken on other kernel sources."""
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
    except Exception:
        return None, "no profiles/ncu_traffic.json"
    ent = tr.get(key)
    if not ent:
        return None, f"no ncu capture for {key}"
    if ent.get("_source_hash") != kernel_source_hash():
        return None, f"stale ncu capture for {key} (kernel sources changed since)"
    return {k: v for k, v in ent.items() if not k.startswith("_")}, ent.get("_captured")


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu, self.rows, self.proc = gpu_index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        sms = [float(r[0]) for r in self.rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nm in enumerate(names):
                if len(r) > 4 + i and r[4 + i].lower().startswith("active"):
                    reasons.add(nm)
        sms.sort()
        return {"sm_mhz": sms[len(sms) // 2] if sms else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sms)}


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


# ----------------------------------------------------------------------------- CPU oracle
def oracle_sample(w, scale):
    """A bounded sample of the same workload recipe (Kronecker at 2^scale, same ef/k/heads)."""
    from paper_conf_sc_bestarglzcgssci23_b200 import gen
    ef = max(1, w.n_samples // w.n)
    n = 1 << scale if w.graph != "er" else min(w.n, 1 << scale)
    import dataclasses
    return dataclasses.replace(w, name=f"{w.name}-sample-2^{scale}", scale=scale, n=n,
                               n_samples=ef * n)


def time_oracle(w, scale, reps=1):
    sys.path.insert(0, os.path.join(ROOT, "oracle"))
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import oracle
    import parity_utils as pu
    ws = oracle_sample(w, scale)
    src, dst = ws.host_edges()
    rp, ci = oracle.csr_build(ws.n, src, dst)
    H, Ws, As, R = ws.host_inputs()
    times = []
    for _ in range(reps):
        t0 = time.perf_counter()
        oracle_train_step(pu, ws, rp, ci, H, Ws, As, R)
        times.append(time.perf_counter() - t0)
    return ws, len(ci), times, oracle_threads()


def oracle_threads():
    """OpenMP threads the oracle's libgomp runs with (the cores it actually uses)."""
    import ctypes
    try:
        return int(ctypes.CDLL("libgomp.so.1").omp_get_max_threads())
    except Exception:
        return len(os.sched_getaffinity(0))


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def workload(args, world=1):
    from paper_conf_sc_bestarglzcgssci23_b200 import gen
    w = gen.CONFIGS[args.config]
    if getattr(args, "weak", False) and w.graph != "er":
        import dataclasses
        ef = w.n_samples // w.n
        n = (1 << 21) * world
        if n & (n - 1):
            sys.exit("bench.py --weak: the Kronecker recipe needs a power-of-two number of GPUs")
        w = dataclasses.replace(w, name=f"{w.name}-weak{world}", scale=n.bit_length() - 1,
                                n=n, n_samples=ef * n)
    if getattr(args, "prec", "fp32") != "fp32":
        import dataclasses
        w = dataclasses.replace(w, prec=args.prec)
    if args.scale is not None and w.graph != "er":
        ef = w.n_samples // w.n
        import dataclasses
        w = dataclasses.replace(w, name=f"{w.name}@2^{args.scale}", scale=args.scale,
                                n=1 << args.scale, n_samples=ef << args.scale)
    return w


def metric_name(w):
    if w.train:
        return f"{w.model.upper()} training step (fwd+bwd+SGD) edges/s"
    return METRIC if w.model == "gat" else f"{w.model.upper()} layer fwd+bwd edges/s"


def oracle_train_step(pu, w, rp, ci, H, Ws, As, R):
    """One oracle step; for training workloads also the SGD update (numpy, fp64)."""
    ref = pu.oracle_step(w, rp, ci, H, Ws, As, R)
    if w.train:
        for l in range(w.layers):
            Ws[l] = Ws[l] - w.lr * ref["dW"][l]
            if As[l] is not None:
                As[l] = As[l] - w.lr * ref["da"][l]
    return ref


def run_reference(args):
    """--impl reference: the FP64 oracle (this tier's reference arm) on host cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    if "WORLD_SIZE" in os.environ:  # torchrun sets OMP_NUM_THREADS=1; the oracle uses every core
        os.environ["OMP_NUM_THREADS"] = str(len(os.sched_getaffinity(0)))
    from paper_conf_sc_bestarglzcgssci23_b200 import gen
    w = workload(args, int(os.environ.get("WORLD_SIZE", str(args.gpus))))
    ws = oracle_sample(w, args.cpu_sample_scale)
    sys.path.insert(0, os.path.join(ROOT, "oracle"))
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import oracle
    import parity_utils as pu
    src, dst = ws.host_edges()
    rp, ci = oracle.csr_build(ws.n, src, dst)
    H, Ws, As, R = ws.host_inputs()
    for _ in range(args.warmup):
        oracle_train_step(pu, ws, rp, ci, H, Ws, As, R)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle_train_step(pu, ws, rp, ci, H, Ws, As, R)
    T = (time.perf_counter() - t0) / args.steps
    m = len(ci)
    val = ws.layers * m / T
    cores = oracle_threads()
    sample = (f"oracle (C, FP64, OpenMP) on {gen.describe(ws)}, m={m} — a bounded sample of "
              f"{args.config} ({gen.describe(w)})")
    line = {"impl": "reference", "metric": metric_name(w), "value": val, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": T * 1e3,
            "higher_is_better": True, "scaling": "weak" if args.weak else "strong",
            "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": args.config, "model": w.model, "graph": w.graph,
                       "n": ws.n, "edges": m, "k": w.k, "heads": w.heads, "layers": w.layers,
                       "sample_of": gen.describe(w)},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": sample, "cpu": cpu_model()},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- ours
def gat_factored(w, mode=1):
    """The factored GAT backward (gat_args.cuh) on symmetric patterns: plan option
    gat_factored (include/agnn.h) = 1 (default): k' = 128; 2: every width; 0: never."""
    k128 = w.k == 128 and w.heads in (1, 2, 4, 8)
    return w.model == "gat" and (mode == 2 or (mode == 1 and k128))


def pass_bytes(w, m, n, factored_mode=1):
    """Algorithmic bytes of each sparse pass per launch:
    {pass: (bytes, per stored edge, per row)}.  f = stored feature bytes (bf16 P, G
    in BF16 mode, reading B1); outputs and dP are fp32.

    GAT forward, per edge: 4 B column index + the gathered P_j row + t_j (4 h);
      per row: s_i (4 h), Z_i and H_out_i written (2 k' 4), Q_i written when the
      backward is factored (k' 4), m, l (8 h), row_ptr (8).
    GAT backward, factored: per edge 4 + the gathered G_i row + rec_i (16 h); per
      row P_j read, dP_j written, ds_j and t_j (8 h), row_ptr.
    GAT backward, unfactored: per edge 4 + P_i and G_i rows + rec_i and t_i
      (20 h); per row P_j, G_j read, dP_j written, record + t (20 h), row_ptr.
    AGNN/VA backward: per edge 4 + 2 k f (+16 AGNN record); per row H_j, M_j read,
      dH_j written (3 k f) (+16) + 8.  BF16 storage (reading B2): H~, M~ rows are
      2 k bytes (dH stays fp32).
    """
    f = 4
    out = {}
    if w.model == "gat":
        fs = 2 if w.prec == "bf16" else 4
        fac = gat_factored(w, factored_mode)
        pe = 4 + w.k * fs + 4 * w.heads
        pr = 4 * w.heads + (3 if fac else 2) * w.k * f + 8 * w.heads + 8
        out["fwd"] = (pe * m + pr * n, pe, pr)
        if fac:
            pe, pr = 4 + w.k * fs + 16 * w.heads, w.k * fs + w.k * f + 8 * w.heads + 8
        else:
            pe, pr = 4 + 2 * w.k * fs + 20 * w.heads, 2 * w.k * fs + w.k * f + 20 * w.heads + 8
        out["bwd"] = (pe * m + pr * n, pe, pr)
    else:
        fs = 2 if w.prec == "bf16" else 4
        rec = 16 if w.model == "agnn" else 0
        pe, pr = 4 + 2 * w.k * fs + rec, 2 * w.k * fs + w.k * f + rec + 8
        out["bwd"] = (pe * m + pr * n, pe, pr)
    return out


# the launches of each sparse pass: the row kernel plus, where the plan splits rows by
# degree, the short-row kernel (both cover the edges of pass_bytes together)
PASSES = {"gat": {"bwd": ("gat_bwd_kernel", "gat_bwd_short_kernel"),
                  "fwd": ("gat_fwd_kernel", "gat_fwd_short_kernel")},
          "agnn": {"bwd": ("av_bwd_kernel",)}, "va": {"bwd": ("av_bwd_kernel",)}}


def roofline(args, w, st, prof, world):
    """Roofline object of the dominant sparse pass (largest share of the step) from the
    live per-kernel event profile; every sparse pass is listed under "passes".

    frac = ncu DRAM bytes per launch (committed capture of the same kernels on the
    same workload, refused when stale) / live launch time / measured HBM peak —
    S§8(d)'s "HBM roofline fraction"; model_frac = algorithmic bytes / time / peak;
    gather_peak_frac = DRAM rate / the measured random-row gather rate."""
    peaks = measured_peaks()
    hbm = peaks.get("hbm_gbs")
    peak_src = ("measured (MEASURED_PEAKS.json hbm_gbs, copy; the burst figure: each pass is "
                "timed as its own launches)" if hbm else "fallback (B200_PROFILING.md)")
    hbm = hbm or 6650.0
    step_ms_prof = sum(v[1] for v in prof.values()) / args.steps
    key = args.config + ("" if w.prec == "fp32" else "-" + w.prec)
    if args.scale is not None or world > 1 or getattr(args, "weak", False):
        per, why = None, "no ncu capture for this workload / world size"
    else:
        per, why = ncu_traffic(key)
    passes = {}
    pb = pass_bytes(w, st.nnz_local, st.n_local)
    for pname, kernels in PASSES.get(w.model, {}).items():
        names = [k for k in kernels if k in prof]
        if not names or pname not in pb:
            continue
        cnt = prof[names[0]][0]
        tot = sum(prof[k][1] for k in names)
        alg, per_edge, per_row = pb[pname]
        ms = tot / cnt if cnt else None  # the pass per layer (its launches back to back)
        model = (alg / (ms / 1e3) / 1e9) if ms else None
        traffic = sum(per[k] for k in names) if per and all(k in per for k in names) else None
        dram = (traffic / (ms / 1e3) / 1e9) if (traffic and ms) else None
        passes[pname] = {
            "bound": "hbm", "kernel": "+".join(names),
            "achieved": dram, "peak": hbm, "unit": "GB/s",
            "frac": (dram / hbm) if dram else None, "traffic": traffic,
            "achieved_basis": ("ncu DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) per "
                               "launch / live CUDA-event launch time") if dram else why,
            "model_achieved": model, "model_frac": (model / hbm) if model else None,
            "gather_peak_gbs": GATHER_PEAK_GBS,
            "gather_peak_frac": (dram / GATHER_PEAK_GBS) if dram else None,
            "peak_source": peak_src, "algorithmic_bytes_per_launch": alg,
            "bytes_per_edge": per_edge, "bytes_per_row": per_row, "launch_ms": ms,
            "share_of_step": (tot / args.steps / step_ms_prof) if step_ms_prof else None}
    if not passes:
        return None
    dom = max(passes, key=lambda k: passes[k]["share_of_step"] or 0)
    r = dict(passes[dom])
    r["pass"] = dom
    r["passes"] = passes
    r["ncu_capture"] = why if per else None
    return r


# dense TF32 : BF16 tensor throughput (B200_PROFILING.md nominal dense peaks: 1.1 and
# 2.25 PFLOP/s); the TF32 peak is the measured BF16 peak times this ratio
TF32_PER_BF16 = 1.1 / 2.25


def gemm_flops_bytes(w, n, spmmm=False):
    """Algorithmic FLOPs (3xTF32: every MMA of the three-term split counted, S§8(d))
    and bytes of the tcgen05 GEMMs of one fwd+bwd step, by profile name.
    GAT: gemm_tc = projection [P|s|t] = H W_ext (N = k' + 2h) + dH = dP W^T;
    gemm_tn = dW = H^T dP.  AGNN / VA: gemm_tc = Z = X W (unless the fused SpMMM
    kernel does it) + M = G W^T; gemm_tn = dW = X^T G.  Bytes: operands read once,
    outputs written once (P~ / M~ two bytes in BF16 storage)."""
    k, L, fs = w.k, w.layers, (2 if w.prec == "bf16" else 4)
    mm = lambda K, N: 3 * 2 * n * K * N  # noqa: E731
    if w.model == "gat":
        tc_f = mm(k, k + 2 * w.heads) + mm(k, k)
        tc_b = n * k * 4 + n * (k * fs + 2 * w.heads * 4) + n * k * 4 + n * k * 4
    else:
        tc_f = mm(k, k) * (1 if spmmm else 2)
        tc_b = n * k * fs + n * k * 4 + (0 if spmmm else n * k * 4 + 2 * n * k * 4)
    tn_f, tn_b = mm(k, k), 2 * n * k * 4
    return {"gemm_tc_kernel": (tc_f * L, tc_b * L), "gemm_tn_kernel": (tn_f * L, tn_b * L)}


def gemm_roofline(args, w, st, prof):
    """The tcgen05 GEMMs against the tensor-pipe peak (TF32) and the HBM peak
    (north_star item 3; S§8(d) "report the GEMMs against HBM (primary) and against
    the tensor pipe (secondary)"), from the live per-kernel event profile."""
    peaks = measured_peaks()
    bf16 = peaks.get("bf16_tflops")
    tpeak = bf16 * TF32_PER_BF16 if bf16 else 1100.0
    hbm = peaks.get("hbm_gbs") or 6650.0
    out = {}
    for name, (fl, by) in gemm_flops_bytes(w, st.n_local, "av_spmmm_kernel" in prof).items():
        if name not in prof:
            continue
        ms = prof[name][1] / args.steps
        tf = fl / (ms / 1e3) / 1e12
        gb = by / (ms / 1e3) / 1e9
        out[name] = {"ms_per_step": ms, "tflops": tf, "tensor_peak_tflops": tpeak,
                     "tensor_frac": tf / tpeak, "hbm_gbs": gb, "hbm_frac": gb / hbm,
                     "flops_per_step": fl, "bytes_per_step": by}
    if not out:
        return None
    out["basis"] = ("3xTF32 FLOPs (three MMAs per product) and operand/output bytes per "
                    "step / live CUDA-event time; tensor peak = MEASURED_PEAKS bf16_tflops "
                    "x 1.1/2.25 (TF32:BF16 dense, B200_PROFILING.md)" if bf16 else
                    "fallback peaks (B200_PROFILING.md)")
    return out


def comm_split(prof, steps):
    """ms per step of the exchange (peer barriers, pushes, reductions or NCCL) and of
    everything else, from the live per-kernel profile of this rank."""
    comm = sum(v[1] for k, v in prof.items() if k.startswith(("peer_", "nccl_")))
    tot = sum(v[1] for v in prof.values())
    return {"comm_ms_per_step": comm / steps, "compute_ms_per_step": (tot - comm) / steps}


def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_sc_bestarglzcgssci23_b200 import agnn, gen, runner

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if not torch.cuda.is_available():
        raise RuntimeError("bench.py needs CUDA GPUs (no CPU fallback)")
    # AGNN_BENCH_SAME_GPU=1 (test only): every rank on cuda:0 with a gloo process group,
    # so the multi-rank bench path runs on a one-GPU box (peer exchange between processes
    # on one device; numbers from such a run are not scaling measurements)
    same_gpu = os.environ.get("AGNN_BENCH_SAME_GPU") == "1"
    if same_gpu:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if same_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    if world != args.gpus and rank == 0:
        print(f"bench: --gpus {args.gpus} but WORLD_SIZE={world}; reporting n_gpus={world}",
              file=sys.stderr)
    w = workload(args, world)
    agnn.lib()
    uid = None
    if world > 1 and args.comm == "peer" and not same_gpu:
        # the peer-memory exchange maps the other GPUs' buffers (CUDA IPC over
        # NVLink): every rank checks P2P access to every other visible GPU, and if
        # any pair lacks it all ranks fall back to the NCCL exchange together
        ok = all(torch.cuda.can_device_access_peer(local, d)
                 for d in range(torch.cuda.device_count()) if d != local)
        flag = torch.tensor([1 if ok else 0], device=dev, dtype=torch.int32)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if int(flag.item()) == 0:
            if rank == 0:
                print("bench: no P2P access between some GPUs; using the NCCL exchange",
                      file=sys.stderr)
            args.comm = "nccl"
    if world > 1 and args.comm == "nccl":
        obj = [agnn.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]

    t_setup = time.perf_counter()
    popts = {"spmmm": args.spmmm} if args.spmmm >= 0 else None
    st = runner.Stack(w, dev, rank=rank, world=world, nccl_uid=uid, plan_options=popts)
    torch.cuda.synchronize()
    setup_s = time.perf_counter() - t_setup
    m, n = st.graph.nnz, w.n
    stream = st.stream

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        st.step()
    barrier()

    # ---- device-resident timed region -----------------------------------------
    # Workloads whose inputs exceed the 126 MB L2 (C3-C5) are timed as one event
    # pair around K back-to-back steps.  Smaller ones (C1, C2) would run from L2:
    # every step is then bracketed by its own event pair with a 256 MB buffer
    # written in between (outside the pairs) to flush L2.
    small = m < 50_000_000
    flush_buf = torch.empty(64 << 20, dtype=torch.float32, device=dev) if small else None

    def timed(run_step):
        if not small:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(args.steps):
                run_step()
            e1.record(stream)
            barrier()
            return e0.elapsed_time(e1)
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(args.steps)]
        for a, b in evs:
            flush_buf.zero_()
            a.record(stream)
            run_step()
            b.record(stream)
        barrier()
        return sum(a.elapsed_time(b) for a, b in evs)

    busy_steps = {}

    def keep_busy(run_step, seconds=0.6):
        # short timed regions (C1, C2: < 1 ms) end before nvidia-smi takes its first
        # sample: keep the GPU under the same load for a moment first, so the clock
        # samples straddle the timed steps.  Every rank must run the same number of
        # steps (the exchange barriers pair up across ranks): the count is fixed from
        # a timed step, the maximum over ranks.
        if not small:
            return
        if seconds not in busy_steps:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            run_step()
            torch.cuda.synchronize()
            cnt = max(1, int(seconds / max(time.perf_counter() - t0, 1e-5)))
            if world > 1:
                c = torch.tensor([cnt], device="cpu" if same_gpu else dev)
                dist.all_reduce(c, op=dist.ReduceOp.MAX)
                cnt = int(c.item())
            busy_steps[seconds] = cnt
        for _ in range(busy_steps[seconds]):
            run_step()
        torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    keep_busy(st.step)
    agnn.profile_enable(True)
    agnn.profile_reset()
    launches0 = agnn.launch_count()
    barrier()
    ms = timed(st.step)
    launches = agnn.launch_count() - launches0
    prof = agnn.profile_report()
    agnn.profile_enable(False)
    if small:
        keep_busy(st.step, 0.25)
    ck = clocks.stop()
    eager_ms = ms
    use_graph = world == 1 and (args.graph == "on" or (args.graph == "auto" and small))
    if use_graph:
        # C1/C2-sized steps are launch-bound (S§8(d)): capture the whole step (all its
        # library launches) once and time graph replays.  The per-kernel profile above
        # (eager, same kernels) still provides the kernel shares and the roofline.
        graph = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream(dev)
        cap.wait_stream(stream)
        with torch.cuda.stream(cap):
            st.stream = cap
            st.step()  # warm the capture stream
            cap.synchronize()
            with torch.cuda.graph(graph, stream=cap):
                st.step()
        st.stream = stream
        stream.wait_stream(cap)
        for _ in range(args.warmup):
            graph.replay()
        barrier()
        clocks = ClockSampler(local)
        clocks.start()
        keep_busy(graph.replay)
        ms = timed(graph.replay)
        keep_busy(graph.replay, 0.25)
        ck = clocks.stop()
    if world > 1:
        t = torch.tensor([ms], device="cpu" if same_gpu else dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    T = ms / 1e3 / args.steps
    value = w.layers * m / T

    # ---- roofline of the dominant kernel ----------------------------------------
    roof = roofline(args, w, st, prof, world)
    groof = gemm_roofline(args, w, st, prof)
    kernels = {k: {"launches": v[0], "ms_per_step": v[1] / args.steps} for k, v in prof.items()}
    split = comm_split(prof, args.steps)
    per_rank = [split]
    if world > 1:
        per_rank = [None] * world
        dist.all_gather_object(per_rank, dict(split, rank=rank, rows=st.n_local,
                                              edges=st.nnz_local))

    # ---- end-to-end through the C ABI with host buffers -------------------------
    # Every step copies its input, the features H^0, from pinned host memory, runs the
    # step through agnn_forward/agnn_backward, evaluates the loss L = <R, H^L>
    # (agnn_loss_inner, reading A13) and reads the step's results back: the loss and
    # the parameter gradients dW (and da).  R is the loss's fixed target tensor
    # (reading A13: a seeded constant of the loss, like W it stays resident on the
    # device), so it is not an input of the step.  Inputs are double-buffered on the
    # device: step s+1's H2D runs on a copy stream while step s computes (input
    # prefetch as a training loop does it); the timed region spans all K steps' copies.
    e2e = None
    if not args.no_e2e:
        nl, k, L = st.n_local, w.k, w.layers
        h_H = torch.empty((nl, k), dtype=torch.float32, pin_memory=True)
        h_loss = torch.empty(1, dtype=torch.float64, pin_memory=True)
        h_dW = [torch.empty(tuple(x.shape), dtype=torch.float32, pin_memory=True) for x in st.dW]
        das = [x for x in st.da if x is not None]
        h_da = [torch.empty(tuple(x.shape), dtype=torch.float32, pin_memory=True) for x in das]
        h_H.copy_(st.H[0].cpu())
        Hb = [st.H[0], torch.empty_like(st.H[0])]
        up, down = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        ev_in = [torch.cuda.Event(), torch.cuda.Event()]
        ev_done = [torch.cuda.Event(), torch.cuda.Event()]
        st.loss()  # allocate the loss buffers outside the timed region
        barrier()
        e2, e3 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e2.record(stream)
        up.wait_stream(stream)
        with torch.cuda.stream(up):
            Hb[0].copy_(h_H, non_blocking=True)
            ev_in[0].record(up)
        for s_ in range(args.steps):
            b = s_ & 1
            if s_ + 1 < args.steps:  # prefetch the next step's input into the other buffer
                with torch.cuda.stream(up):
                    if s_ >= 1:
                        up.wait_event(ev_done[b ^ 1])
                    Hb[b ^ 1].copy_(h_H, non_blocking=True)
                    ev_in[b ^ 1].record(up)
            stream.wait_event(ev_in[b])
            st.H[0] = Hb[b]
            st.step()
            loss_d = st.loss()
            ev_done[b].record(stream)
            with torch.cuda.stream(down):
                down.wait_event(ev_done[b])
                h_loss.copy_(loss_d, non_blocking=True)
                for hw_, dw_ in zip(h_dW, st.dW):
                    hw_.copy_(dw_, non_blocking=True)
                for ha_, da_ in zip(h_da, das):
                    ha_.copy_(da_, non_blocking=True)
            stream.wait_stream(down)  # the next step overwrites dW / da / loss
        stream.wait_stream(up)
        e3.record(stream)
        barrier()
        st.H[0] = Hb[0]
        ms2 = e2.elapsed_time(e3)
        if world > 1:
            t = torch.tensor([ms2], device="cpu" if same_gpu else dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms2 = float(t.item())
        T2 = ms2 / 1e3 / args.steps
        h2d = nl * k * 4
        d2h = 8 + sum(x.numel() * 4 for x in h_dW) + sum(x.numel() * 4 for x in h_da)
        e2e = {"value": w.layers * m / T2, "unit": UNIT, "h2d_bytes_per_step": h2d * world,
               "d2h_bytes_per_step": d2h * world, "ms_per_step": T2 * 1e3,
               "api": "agnn_forward/agnn_backward/agnn_loss_inner via "
                      "paper_conf_sc_bestarglzcgssci23_b200.runner",
               "inputs": "H^0 (features) copied from pinned host memory every step; the loss "
                         "target R (reading A13) is a resident constant of the loss",
               "result_read_back": "loss <R, H^L> (fp64) + dW + da per step",
               "overlap": "double-buffered input: H2D of step s+1 overlaps step s",
               "loss": float(h_loss.item())}

    # ---- CPU oracle baseline (rank 0, N = 1 only) ------------------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        ws_, m_s, times, cores = time_oracle(w, args.cpu_sample_scale)
        t_med = sorted(times)[len(times) // 2]
        cpu = {"value": ws_.layers * m_s / t_med, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"FP64 C oracle fwd+bwd on {gen.describe(ws_)} (m={m_s}), same recipe "
                         f"as {args.config} at 2^{args.cpu_sample_scale} vertices; "
                         f"{t_med:.1f} s", "cpu": cpu_model()}

    # ---- the same workload in the BF16 storage mode (GAT, k' = 128) ----------------
    # north_star: "within 1e-5 relative in FP32 (1e-2 with BF16 projection)".  The
    # headline line above is the FP32 mode; this object is the same step with P and
    # G stored as bfloat16 (include/agnn.h AGNN_PREC_BF16, reading B1: fp32
    # arithmetic, bf16 storage of the gathered rows), device-timed the same way.
    bf16 = None
    bf16_ok = ((w.model == "gat" and w.k == 128) or (w.model in ("agnn", "va") and w.k in (128, 256)))
    if (bf16_ok and w.prec == "fp32" and not args.no_bf16_line
            and uid is None):  # (an NCCL unique id serves one communicator)
        import dataclasses
        w16 = dataclasses.replace(w, prec="bf16")
        graph = st.graph
        st.__dict__.clear()   # free the FP32 buffers (saved, workspace) first
        del st
        torch.cuda.empty_cache()
        s16 = runner.Stack(w16, dev, rank=rank, world=world, nccl_uid=uid, graph=graph)
        stream = s16.stream
        for _ in range(args.warmup):
            s16.step()
        barrier()
        agnn.profile_enable(True)
        agnn.profile_reset()
        l0 = agnn.launch_count()
        barrier()
        ms16 = timed(s16.step)
        l16 = agnn.launch_count() - l0
        prof16 = agnn.profile_report()
        agnn.profile_enable(False)
        if world > 1:
            t = torch.tensor([ms16], device="cpu" if same_gpu else dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms16 = float(t.item())
        bf16 = {"value": w.layers * m / (ms16 / 1e3 / args.steps), "unit": UNIT,
                "ms_per_step": ms16 / args.steps, "dtype": "f32",
                "storage": ("bf16 P, G (fp32 arithmetic; AGNN_PREC_BF16, reading B1)"
                            if w.model == "gat" else
                            "bf16 H, M (fp32 arithmetic; AGNN_PREC_BF16, reading B2)"),
                "tolerance": "1e-2 normwise (north_star 'BF16 projection')",
                "roofline": roofline(args, w16, s16, prof16, world), "gpu_launches": l16,
                "kernels": {k: {"launches": v[0], "ms_per_step": v[1] / args.steps}
                            for k, v in prof16.items()}}

    if rank == 0:
        line = {"metric": metric_name(w),
                "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": T * 1e3, "higher_is_better": True,
                "scaling": "weak" if args.weak else "strong", "vs_baseline": None,
                "dtype": "f32", "data": "synthetic",
                "config": {"workload": args.config, "model": w.model, "graph": w.graph,
                           "n": n, "edges": m, "k": w.k, "heads": w.heads, "layers": w.layers,
                           "storage": ("bf16 gathered rows (fp32 arithmetic; AGNN_PREC_BF16, "
                                       "tol 1e-2)" if w.prec == "bf16" else "fp32"),
                           "parallelism": f"1d-rowblock{world}",
                           "comm": (args.comm if world > 1 else None),
                           "l2_flush": "inputs > L2 (126 MB)" if not small else
                                       "256 MB buffer written between timed steps (per-step "
                                       "event pairs)",
                           "cuda_graph": use_graph, "eager_ms_per_step": eager_ms / args.steps,
                           "spmmm": (args.spmmm if args.spmmm >= 0 else "library default")
                                    if w.model in ("agnn", "va") and w.k == 128 else None,
                           "setup_s": setup_s},
                "roofline": roof, "gemm_roofline": groof,
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
                "clocks": ck, "kernels": kernels, "per_rank": per_rank}
        if same_gpu and world > 1:
            line["note"] = ("AGNN_BENCH_SAME_GPU: every rank ran on cuda:0 (functional test of the "
                            "multi-rank path, not a scaling measurement)")
        if bf16 is not None:
            line["bf16_storage"] = bf16
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    maybe_relaunch(args)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
