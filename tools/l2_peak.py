"""L2-atomic peak microbenchmark (the roofline denominator).

Runs every pattern of ga_l2_atomic_bench (include/ga_bench.h) on a full grid
(148 x 8 blocks of 256) and times it with CUDA events.  With --ncu-csv it instead
reads an ncu capture of the same command (metrics lts__t_requests_op_atom.sum,
lts__t_requests_op_red.sum, gpu__time_duration.sum) and writes the committed
denominator profiles/l2_atomic_peak.json: the event-timed distinct-word peak,
cross-checked against ncu's L2 atomic / reduction request counts per launch.

usage (GPU box):  python tools/l2_peak.py > gpurun_out/l2_live.json
                  ncu --metrics lts__t_requests_op_atom.sum,lts__t_requests_op_red.sum,gpu__time_duration.sum \
                      --csv --log-file gpurun_out/l2_ncu.csv python tools/l2_peak.py --reps 1
here:             python tools/l2_peak.py --ncu-csv gpurun_out/l2_ncu.csv --live gpurun_out/l2_live.json
"""
import argparse
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
GRID, BLOCK = 148 * 8, 256
NAMES = {0: "atomg_distinct", 1: "redg_distinct", 2: "atomg_hot_word", 3: "atomg_1184_words",
         4: "cas_distinct", 5: "cas_148_words"}
ITERS = {0: 64, 1: 64, 2: 4, 3: 16, 4: 16, 5: 2}


def live(reps):
    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    torch.cuda.set_device(0)
    s = torch.cuda.current_stream()
    buf = torch.zeros(GRID * BLOCK * 4 + 8192, dtype=torch.int64, device="cuda")
    sink = torch.zeros(8, dtype=torch.int64, device="cuda")
    out = {}
    for pat, name in NAMES.items():
        best = None
        for rep in range(reps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            ga.ga_l2_atomic_bench(s.cuda_stream, pat, buf.data_ptr(), buf.numel(), ITERS[pat], GRID, BLOCK,
                                  sink.data_ptr())
            e1.record(s)
            e1.synchronize()
            if rep:
                t = e0.elapsed_time(e1) / 1e3
                best = t if best is None else min(best, t)
        ops = GRID * BLOCK * ITERS[pat]
        out[name] = {"ops_per_launch": ops, "seconds": best, "gatom_s": ops / best / 1e9 if best else None}
    return out


def summarise(ncu_csv, live_json):
    rows = list(csv.DictReader(l for l in open(ncu_csv) if not l.startswith("==")))
    per = {}
    for r in rows:
        if "k_l2_atomic" not in r.get("Kernel Name", ""):
            continue
        per.setdefault(int(r["ID"]), {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    launches = [per[k] for k in sorted(per)]
    lv = json.load(open(live_json))
    res = {}
    for (pat, name), m in zip(NAMES.items(), launches):        # tools/l2_peak.py launches patterns in order
        ops = GRID * BLOCK * ITERS[pat]
        req = m.get("lts__t_requests_op_atom.sum", 0) + m.get("lts__t_requests_op_red.sum", 0)
        dur = m.get("gpu__time_duration.sum", 0) / 1e9
        res[name] = {"ops_per_launch": ops, "ncu_l2_atom_red_requests": req, "requests_per_op": req / ops,
                     "ncu_duration_s": dur, "ncu_gatom_s": ops / dur / 1e9 if dur else None,
                     "event_gatom_s": lv[name]["gatom_s"]}
    peak_name = max(("atomg_distinct", "redg_distinct"), key=lambda n: lv[n]["gatom_s"])
    out = {"peak_gatom_s": round(lv[peak_name]["gatom_s"], 1),
           "source": f"profiles/l2_atomic_peak.json: {peak_name}, 148x8x256 threads, event-timed; "
                     f"ncu L2 atom+red requests per op = {res[peak_name]['requests_per_op']:.3f}",
           "patterns": res}
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--ncu-csv")
    ap.add_argument("--live")
    a = ap.parse_args()
    if a.ncu_csv:
        out = summarise(a.ncu_csv, a.live)
        json.dump(out, open(os.path.join(ROOT, "profiles", "l2_atomic_peak.json"), "w"), indent=1)
        print(json.dumps(out, indent=1))
    else:
        print(json.dumps(live(a.reps)))
