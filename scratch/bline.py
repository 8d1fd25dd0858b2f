"""Print the headline numbers of a bench JSON line (scratch helper)."""
import json, sys
for f in sys.argv[1:]:
    lines = [l for l in open(f) if l.startswith("{")]
    if not lines:
        print(f, "no JSON"); continue
    d = json.loads(lines[-1])
    print(f, f"value {d['value']:.3e}  ms {d['ms_per_step']:.2f}  e2e {d['e2e']['value'] if d.get('e2e') else None}")
    r = d.get("roofline") or {}
    print("  roofline", {k: r.get(k) for k in ("pass", "frac", "model_frac", "launch_ms", "share_of_step")})
    print("  clocks", d.get("clocks"))
    print("  ", {k: round(v["ms_per_step"], 2) for k, v in d["kernels"].items() if v["ms_per_step"] > 0.05})
    if d.get("bf16_storage"):
        print("  bf16", f"{d['bf16_storage']['value']:.3e}")
