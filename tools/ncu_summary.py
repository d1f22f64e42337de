"""Summarise an ncu report: key section metrics + stall samples by CUDA source line."""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
want = {"Duration", "Registers Per Thread", "Achieved Occupancy", "Theoretical Occupancy", "Avg. Active Threads Per Warp",
        "L2 Cache Throughput", "DRAM Throughput", "Issue Slots Busy", "No Eligible", "L1/TEX Hit Rate", "L2 Hit Rate",
        "Warp Cycles Per Issued Instruction", "Memory Throughput"}
for r in csv.DictReader(io.StringIO(out)):
    if r.get("Metric Name") in want:
        print(f"  {r['Metric Name']:38s} {r['Metric Value']:>14s} {r['Metric Unit']}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
if len(rows) >= 3:
    h, u, v = rows[0], rows[1], rows[2]
    for name in ("lts__t_requests_op_atom.sum", "lts__t_requests_op_red.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
                 "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "smsp__inst_executed.sum",
                 "gpu__time_duration.sum"):
        if name in h:
            i = h.index(name)
            print(f"  {name:38s} {v[i]:>14s} {u[i]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"]
if hi:
    h = rows[hi[0]]
    si = h.index("Warp Stall Sampling (All Samples)")
    agg, txt = collections.Counter(), {}

    def f(x):
        try:
            return float(x)
        except ValueError:
            return 0.0
    for r in rows[hi[0] + 1:]:
        if len(r) > si and r[0] not in ("", "-"):
            agg[r[0]] += f(r[si])
            txt[r[0]] = r[1]
    tot = sum(agg.values()) or 1
    print(f"  stall samples: {int(tot)}")
    for ln, n in agg.most_common(top):
        print(f"  {100 * n / tot:5.1f}%  L{ln}: {txt[ln].strip()[:100]}")
