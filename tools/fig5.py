"""the paper's Fig. 5 experiment on one B200.

Upper-limit allocation rate of two-stage resource allocation: every thread
acquires ONE unit from a batch of B = 512 (the UAlloc batch) and
never releases it; a thread that finds the semaphore empty produces a new
batch with one atomic on a bump counter.  One semaphore for the
whole grid, as in the paper.  Swept over the number of concurrent threads
(multiple waves above the 303,104 resident threads), for
  counting  -- the growable counting semaphore of Sec. 3.2,
  bulk      -- Alg. 1 / Alg. 2 per thread, exact form (one CAS decides each wait),
  bulk_fa   -- Alg. 1 / Alg. 2 per thread, fetch-add form (each update one
               fetch-add: the paper's "updates to R saturate the atomic
               throughput"),
  bulk_warp -- Alg. 1 / Alg. 2 with one wait per warp for the warp's N units
               (this build's warp aggregation, subsystem 1 of the north star).
Each point checks the acquire-only accounting: every grant is backed, C =
units produced - units granted and D = 0 at the end, and (pin P-2) batches
produced = ceil(threads / B) exactly for the CAS forms; the fetch-add form may
over-produce, and its batches / minimum ratio is reported.
Block sizes: 256 (primary) and, with --all-blocks, the paper's average over
power-of-two blocks 1..1024.

  python tools/fig5.py [--all-blocks] [--out profiles/r01_fig5.json]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

THREADS = [1024, 4096, 16384, 65536, 131072, 262144, 303104, 393216, 524288, 606208]
NAMES = {2: "counting", 1: "bulk", 4: "bulk_fa", 0: "bulk_warp"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--all-blocks", action="store_true")
    ap.add_argument("--B", type=int, default=512)
    ap.add_argument("--out", default=None)
    ap.add_argument("--reps", type=int, default=3, help="timed runs per point (best kept)")
    a = ap.parse_args()
    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream().cuda_stream
    sems = torch.zeros(64, dtype=torch.int64, device="cuda")
    out = torch.zeros(8, dtype=torch.int64, device="cuda")
    blocks = [1 << i for i in range(11)] if a.all_blocks else [256]
    rows = []
    for T in THREADS:
        row = {"threads": T}
        for v in (2, 1, 4, 0):
            per_block = {}
            for blk in blocks:
                grid = (T + blk - 1) // blk
                cfg = ga.BsemCfg(variant=v, k=1, B=a.B, n_sems=1, iters=1, acquire_only=1, grid=grid, block=blk,
                                 seed=0)
                best, ok, over = None, True, 1.0
                for rep in range(a.reps):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    ga.ga_bsem_bench(st, cfg, sems.data_ptr(), out.data_ptr())
                    e1.record()
                    e1.synchronize()
                    t = e0.elapsed_time(e1) / 1e3
                    best = t if best is None else min(best, t)
                    o = out.cpu().numpy()
                    n = grid * blk
                    batches = -(-n // a.B)
                    # exact accounting: every grant backed, C = produced - granted, D = 0;
                    # batches == ceil(n / B) is exact for the CAS forms, the fetch-add
                    # form may over-produce (reported as a ratio)
                    ok &= bool(o[0] == n and o[4] == int(o[3]) - n and o[5] == 0 and o[2] >= batches
                               and (v == 4 or o[2] == batches))
                    over = max(over, float(o[2]) / batches)
                per_block[str(blk)] = {"seconds": best, "allocs_per_s": grid * blk / best, "invariants_ok": ok,
                                       "batches_over_minimum": over}
            vals = list(per_block.values())
            row[NAMES[v]] = {"allocs_per_s_block256": per_block.get("256", vals[0])["allocs_per_s"],
                             "allocs_per_s_avg_time": T / (sum(x["seconds"] for x in vals) / len(vals)),
                             "invariants_ok": all(x["invariants_ok"] for x in vals), "per_block": per_block}
        rows.append(row)
        print(f"T={T:>7d}  " + "  ".join(f"{NAMES[v]} {row[NAMES[v]]['allocs_per_s_block256']:.3e}/s"
                                         f"{'' if row[NAMES[v]]['invariants_ok'] else ' (INVARIANT FAIL)'}"
                                         for v in (2, 1, 4, 0)), flush=True)
    res = {"experiment": "Fig. 5 (P:L1324-1402): acquire-only, one unit per thread, B = %d, one semaphore" % a.B,
           "blocks": blocks, "rows": rows}
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
