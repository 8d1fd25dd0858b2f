"""Key ncu --set full metrics per kernel of a report (details page)."""
import csv, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "details", "--csv"], capture_output=True,
                     text=True).stdout
r = list(csv.reader(out.splitlines()))
hdr = r[0]
ki, mi, vi, ui = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
want = ["Duration", "DRAM Throughput", "Memory Throughput", "L2 Hit Rate", "L1/TEX Hit Rate",
        "Compute (SM) Throughput", "Achieved Occupancy", "Theoretical Occupancy", "Registers Per Thread",
        "Issue Slots Busy", "Executed Ipc Active", "No Eligible", "Active Warps Per Scheduler",
        "Eligible Warps Per Scheduler", "Warp Cycles Per Issued Instruction", "Mem Busy",
        "Max Bandwidth", "Mem Pipes Busy", "L2 Cache Throughput", "L1/TEX Cache Throughput"]
seen = set()
for row in r[1:]:
    key = (row[ki][:60], row[mi], row[ui])
    if row[mi] in want and key not in seen:
        seen.add(key)
        print(f"{row[ki][:50]:50s} | {row[mi]:36s} {row[vi]} {row[ui]}")
