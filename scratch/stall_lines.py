"""Map ncu per-SASS stall samples (source page csv) to CUDA source lines via nvdisasm -g.
usage: stall_lines.py <src.csv> <cubin> <mangled-function-substring> [n]"""
import csv, re, subprocess, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hi]
data = [r for r in rows[hi + 1:] if len(r) == len(hdr) and r[0].startswith("0x")]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
f = lambda x: float(x.replace(",", "")) if x and x[0].isdigit() else 0.0
samples = collections.OrderedDict()
for r in data:
    samples.setdefault(int(r[0], 16), f(r[i_s]))
base = min(samples)
# nvdisasm with line info
dis_all = subprocess.run(["nvdisasm", "-g", sys.argv[2]], capture_output=True, text=True).stdout
secs = re.split(r"\n\s*\.section\s+\.text\.", dis_all)
dis = next(sec for sec in secs if sys.argv[3] in sec.split("\n", 1)[0])
line = None
off2line = {}
for l in dis.splitlines():
    m = re.search(r'//## File ".*?/([^/"]+)", line (\d+)', l)
    if m:
        line = f"{m.group(1)}:{m.group(2)}"
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m:
        off2line[int(m.group(1), 16)] = line
tot = sum(samples.values())
agg = collections.Counter()
for a, v in samples.items():
    agg[off2line.get(a - base, "?")] += v
n = int(sys.argv[4]) if len(sys.argv) > 4 else 25
for k, v in agg.most_common(n):
    print(f"{v / tot * 100:5.1f}%  {k}")
