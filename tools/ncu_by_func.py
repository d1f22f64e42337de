"""Attribute an ncu report's per-SASS-instruction stall samples and executed
instructions to the device functions of the kernel (via the cubin symbol table):
which callee the time goes to.  usage: ncu_by_func.py REP CUBIN KERNEL_SUBSTR"""
import csv
import io
import re
import subprocess
import sys

rep, cubin, ksub = sys.argv[1:4]
syms = []
for ln in subprocess.run(["readelf", "-sW", cubin], capture_output=True, text=True).stdout.splitlines():
    f = ln.split()
    if len(f) >= 8 and f[3] == "FUNC" and ksub in f[7]:
        name = f[7]
        short = re.sub(r".*_ga_bench_cu_[0-9a-f]+\d+ga\d+", "", name.split("$")[-1]) if "$" in name else "<kernel>"
        short = re.sub(r"EPK7ga_desc.*|ENS0_.*", "", short)
        if "bsem_wait_impl" in name:
            short = "bsem_wait_impl<" + ("exact" if "ILb1" in name else "opt") + ("," + "ArenaSpin" if "ArenaSpin" in name else "") + ">"
        syms.append((int(f[1], 16), int(f[2]), short))
syms.sort()
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
ia, iss, iex = h.index("Address"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
base = int(rows[2][ia], 16)
agg = {}
for r in rows[2:]:
    if len(r) <= iex:
        continue
    off = int(r[ia], 16) - base
    fn = "?"
    for v, sz, nm in syms:
        if v <= off < v + max(sz, 1):
            fn = nm
    a = agg.setdefault(fn, [0, 0, 0])
    a[0] += float(r[iss] or 0); a[1] += float(r[iex] or 0); a[2] += 16
ts = sum(a[0] for a in agg.values()) or 1
ti = sum(a[1] for a in agg.values()) or 1
print(f"{'function':36s} {'stall%':>7s} {'inst%':>7s} {'code KB':>8s}")
for fn, a in sorted(agg.items(), key=lambda kv: -kv[1][0]):
    print(f"{fn:36s} {100 * a[0] / ts:7.1f} {100 * a[1] / ti:7.1f} {a[2] / 1024:8.1f}")
