"""Rank SASS instructions of an ncu --page source --csv dump by warp-stall samples."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hi]
data = [r for r in rows[hi + 1:] if len(r) == len(hdr) and r[0] != "Address"]
i_s = hdr.index("Warp Stall Sampling (All Samples)"); i_src = hdr.index("Source"); i_a = hdr.index("Address")
f = lambda x: float(x.replace(",", "")) if x and x[0].isdigit() else 0.0
tot = sum(f(r[i_s]) for r in data)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
for r in sorted(data, key=lambda r: -f(r[i_s]))[:n]:
    print(f"{f(r[i_s]) / tot * 100:5.1f}% {r[i_a]} {r[i_src][:100]}")
