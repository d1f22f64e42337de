"""Summarise tools/r02_coll_ncu.sh's ncu CSVs (gpurun_out/coll_ncu_s{scope}_{workload}.csv)
into profiles/r02_coll_ncu.json: L2 atomic + reduction requests per allocator call,
instructions, active lanes and kernel time per call scope."""
import csv
import glob
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CALLS = 16 * 303104 * 2                      # every workload: 16 rounds x 303,104 threads x (malloc + free)
SCOPE = {0: "warp (ga_malloc)", 1: "block (ga_malloc_block)", 2: "cluster of 2 (ga_malloc_cluster)",
         4: "cluster of 4 (ga_malloc_cluster)"}
out = {"what": "ncu --metrics on the timed kernel (tools/profile_trace.py, one launch after a warm-up launch), "
               "per call scope; calls = 16 rounds x 303,104 threads x 2", "rows": []}
for f in sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "coll_ncu_s*_*.csv"))):
    m = re.search(r"coll_ncu_s(\d+)_(\w+)\.csv", f)
    sc, wl = int(m.group(1)), m.group(2)
    rows = list(csv.reader(ln for ln in open(f) if ln.startswith('"')))
    if not rows:
        continue
    h = rows[0]
    v = {r[h.index("Metric Name")]: float(r[h.index("Metric Value")].replace(",", "")) for r in rows[1:]}
    atom = v.get("lts__t_requests_srcunit_tex_op_atom_dot_alu.sum", 0) + v.get("lts__t_requests_srcunit_tex_op_atom_dot_cas.sum", 0)
    red = v.get("lts__t_requests_srcunit_tex_op_red.sum", 0)
    out["rows"].append({"scope": sc, "scope_name": SCOPE.get(sc, str(sc)), "workload": wl,
                        "ms": v.get("gpu__time_duration.sum", 0) / 1e6,
                        "l2_atomics_per_call": (atom + red) / CALLS, "atom": atom, "red": red,
                        "warp_inst_per_call": v.get("smsp__inst_executed.sum", 0) / CALLS,
                        "active_lanes_per_inst": v.get("smsp__thread_inst_executed_per_inst_executed.ratio"),
                        "regs": v.get("launch__registers_per_thread")})
json.dump(out, open(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02_coll_ncu.json"), "w"), indent=1)
for r in out["rows"]:
    print(f"{r['workload']:7s} scope {r['scope']}  {r['ms']:6.2f} ms  L2 atomics/call {r['l2_atomics_per_call']:.3f}  "
          f"inst/call {r['warp_inst_per_call']:.1f}  lanes {r['active_lanes_per_inst']}")
