"""Summarise an ncu launch list (gpu__time_duration + DRAM bytes per launch) of one
bench step into profiles/<round>_launches_<cfg>_summary.md and update
profiles/ncu_traffic.json (DRAM bytes per launch keyed by the library's kernel
names, which bench.py uses for roofline.traffic), stamped with the hash of the
kernel sources (bench.py refuses an entry whose hash no longer matches).

    python profiles/summarize_launches.py <launches.csv> <config key> <round> <out.md> profiles/ncu_traffic.json
"""
import collections
import csv
import datetime
import importlib.util
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod

ALIAS = {"gat_bwd_k128_kernel": "gat_bwd_kernel", "gat_bwd_k128f_kernel": "gat_bwd_kernel",
         "gat_bwd_short_f_kernel": "gat_bwd_short_kernel",
         "gat_bwd_bundle_kernel": "gat_bwd_short_kernel", "gat_fwd_bundle_kernel": "gat_fwd_short_kernel", "gat_fwd_k128_kernel": "gat_fwd_kernel",
         "gat_fwd_k128_pair_kernel": "gat_fwd_kernel", "gat_bwd_k128f_pair_kernel": "gat_bwd_kernel",
         "av_spmmm_kernel": "av_spmmm_kernel",
                  "av_bwd_k128_kernel": "av_bwd_kernel", "av_fwd_k128_kernel": "av_fwd_kernel",
         "av_bwd_batched_kernel": "av_bwd_kernel", "av_fwd_batched_kernel": "av_fwd_kernel",
         "gemm_tn_tc_kernel": "gemm_tn_kernel", "tn_sum_kernel": "sum_splits_kernel",
         "gemm_tc_roles_kernel": "gemm_tc_kernel"}
STEP = re.compile(r"(gat_|av_|gemm_|agnn_rec|nu_kernel|grad_act|sum_splits|tn_sum|sgd|transpose|to_bf16|cg_)")


def short(name):
    base = name.split("(")[0]
    base = re.sub(r"^void ", "", base)
    m = re.search(r"([A-Za-z0-9_]+)(<[^()]*>)?$", base)
    return (m.group(1), m.group(2) or "") if m else (base, "")


def main(csv_path, cfg, rnd, out_md, traffic_json):
    text = open(csv_path).read().splitlines()
    start = next(i for i, l in enumerate(text) if l.startswith('"ID"'))
    rows = list(csv.DictReader(text[start:]))
    per = collections.OrderedDict()
    for r in rows:
        per.setdefault(r["ID"], {"name": r["Kernel Name"]})[r["Metric Name"]] = float(
            r["Metric Value"].replace(",", ""))
    agg = collections.OrderedDict()
    for k in per.values():
        nm, tmpl = short(k["name"])
        key = nm + tmpl
        a = agg.setdefault(key, {"n": 0, "ms": 0.0, "dram": 0.0, "lib": ALIAS.get(nm, nm)})
        a["n"] += 1
        a["ms"] += k.get("gpu__time_duration.sum", 0) / 1e6
        a["dram"] += k.get("dram__bytes_read.sum", 0) + k.get("dram__bytes_write.sum", 0)
    lines = [f"# {rnd} launch list — {cfg}",
             "", "`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
             "--clock-control none python bench.py --config " + cfg +
             " --steps 1 --warmup 1 --no-e2e --no-cpu-baseline` (raw: `" + csv_path.split('/')[-1] + "`).",
             "Includes setup (generation, CSR build, plan) and 2 steps (1 warm-up + 1 timed); serialised, "
             "cold-cache launches, so per-launch times are upper bounds — the SHARE of the step is what "
             "must agree with the live CUDA-event profile in the bench line.", "",
             "| kernel | launches | total ms | ms/launch | DRAM GB/launch | DRAM GB/s |", "|---|---|---|---|---|---|"]
    for key, a in sorted(agg.items(), key=lambda x: -x[1]["ms"]):
        ml = a["ms"] / a["n"]
        gb = a["dram"] / a["n"] / 1e9
        lines.append(f"| `{key[:70]}` | {a['n']} | {a['ms']:.2f} | {ml:.3f} | {gb:.3f} | "
                     f"{(gb / (ml / 1e3)) if ml else 0:.0f} |")
    step = {k: a for k, a in agg.items() if STEP.match(k)}
    tot = sum(a["ms"] / 2 for a in step.values())  # 2 steps in the capture
    lines += ["", "Per-step share of the step kernels (2 steps captured):", ""]
    for key, a in sorted(step.items(), key=lambda x: -x[1]["ms"]):
        lines.append(f"- `{key[:60]}`: {a['ms'] / 2:.2f} ms/step ({a['ms'] / 2 / tot * 100:.1f} %)")
    open(out_md, "w").write("\n".join(lines) + "\n")
    tr = json.load(open(traffic_json)) if traffic_json else {}
    cfgd = {}
    for key, a in step.items():
        cfgd[a["lib"]] = max(cfgd.get(a["lib"], 0.0), a["dram"] / a["n"])
    cfgd["_source_hash"] = _bench().kernel_source_hash()
    cfgd["_captured"] = (f"{rnd} {datetime.date.today().isoformat()}: ncu --metrics "
                         "dram__bytes_read.sum,dram__bytes_write.sum per launch of one bench step "
                         f"({os.path.basename(csv_path)})")
    tr[cfg] = cfgd
    tr["_source"] = ("ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum per launch of one "
                     "bench step (profiles/summarize_launches.py over the launch-list csv)")
    json.dump(tr, open(traffic_json, "w"), indent=1)


if __name__ == "__main__":
    main(*sys.argv[1:6])
