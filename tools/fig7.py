"""the paper's Fig. 7 experiment on one B200.

Each thread makes ONE malloc of a fixed size; just enough threads run to
exhaust the pool, so failures measure fragmentation.  Pool
sizing follows P:L1618-1630: 8 MB at 8 B, growing with the size so 2^20
threads run, up to 512 MB at 512 B; above that the pool stays 512 MB and the
thread count falls (1,024 threads at 512 KiB).  Rates count failed calls
(P:L1646-1648).  Our allocator and CUDA's device malloc run the same trace with
the same pool: ours through ga_trace_phase (malloc phase timed, the free
phase untimed), CUDA's in a fresh process per size because its heap limit can
only be set before the first kernel that uses it.  The oracle's failure count
for the same trace (build layout) is reported beside ours.  Block sizes: 256
(full occupancy, primary) and, with --all-blocks, the paper's average over
power-of-two blocks 1..1024 (reading R-25).

  python tools/fig7.py [--all-blocks] [--out profiles/r01_fig7.json]
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SIZES = [8 << i for i in range(17)]                 # 8 B .. 512 KiB
MB = 1 << 20


def pool_of(s: int) -> int:
    return min(8 * MB * s // 8, 512 * MB)


def blocks_of(all_blocks: bool):
    return [1 << i for i in range(11)] if all_blocks else [256]


def time_phase(run_malloc, run_free, reps: int = 2):
    import torch
    best = None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        run_malloc()
        e1.record()
        e1.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
        run_free()
        torch.cuda.synchronize()
    return best


def one_size(s: int, cuda: bool, all_blocks: bool, reps: int = 2) -> dict:
    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    from paper_conf_ppopp_geladog19_b200.runner import GpuHeap
    torch.cuda.set_device(0)
    pool = pool_of(s)
    T = pool // s
    st = torch.cuda.current_stream().cuda_stream
    if cuda:
        ga.ga_cuda_set_heap_limit(pool)
    heap = None if cuda else GpuHeap(pool)
    d = torch.full((T,), s, dtype=torch.int32, device="cuda")
    held = torch.empty(2 * T, dtype=torch.int64, device="cuda")
    cnt = torch.zeros(8, dtype=torch.int64, device="cuda")
    res = {"size": s, "pool_bytes": pool, "threads": T, "per_block": {}}
    for blk in blocks_of(all_blocks):
        def mal():
            cnt.zero_()
            held[0::2] = -1
            if cuda:
                ga.ga_cuda_trace_phase(st, d.data_ptr(), 1, T, 0, 0, 0, held.data_ptr(), cnt.data_ptr(), 0, blk)
            else:
                ga.ga_trace_phase(heap.h, st, d.data_ptr(), 1, T, 0, 0, 0, held.data_ptr(), 0, cnt.data_ptr(), 0, blk)

        fails = []

        def fre():
            fails.append(int(cnt[1].item()))
            if cuda:
                ga.ga_cuda_trace_phase(st, d.data_ptr(), 1, T, 0, 0, 1, held.data_ptr(), cnt.data_ptr(), 0, blk)
            else:
                ga.ga_trace_phase(heap.h, st, d.data_ptr(), 1, T, 0, 0, 1, held.data_ptr(), 0, cnt.data_ptr(), 0, blk)
                heap.reset()

        t = time_phase(mal, fre, reps)
        res["per_block"][str(blk)] = {"seconds": t, "allocs_per_s": T / t, "failed": max(fails)}
    v = list(res["per_block"].values())
    res["allocs_per_s_block256"] = res["per_block"].get("256", v[0])["allocs_per_s"]
    res["failed_block256"] = res["per_block"].get("256", v[0])["failed"]
    res["allocs_per_s_avg_time"] = T / (sum(x["seconds"] for x in v) / len(v))
    if heap:
        heap.close()
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--all-blocks", action="store_true")
    ap.add_argument("--out", default=None)
    ap.add_argument("--one", type=int, default=0, help="internal: one size in this process")
    ap.add_argument("--cuda", action="store_true", help="internal: CUDA malloc for --one")
    ap.add_argument("--sizes", default=None)
    ap.add_argument("--reps", type=int, default=2, help="timed malloc phases per block size (best kept)")
    ap.add_argument("--run-timeout", type=int, default=1200, help="seconds per (size, allocator) subprocess")
    a = ap.parse_args()
    if a.one:
        print(json.dumps(one_size(a.one, a.cuda, a.all_blocks, a.reps)))
        return 0
    import oracle
    oracle.build()
    sizes = [int(x) for x in a.sizes.split(",")] if a.sizes else SIZES
    rows = []
    for s in sizes:
        row = {"size": s}
        for who in ("ours", "cuda"):
            cmd = [sys.executable, __file__, "--one", str(s)] + (["--cuda"] if who == "cuda" else []) + \
                  (["--all-blocks"] if a.all_blocks else []) + ["--reps", str(a.reps)]
            try:
                r = subprocess.run(cmd, capture_output=True, text=True, timeout=a.run_timeout)
                lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
                row[who] = json.loads(lines[-1]) if lines else {"error": (r.stderr or "")[-400:]}
            except subprocess.TimeoutExpired:
                row[who] = {"error": f"timed out after {a.run_timeout} s"}
        T, pool = pool_of(s) // s, pool_of(s)
        ref = oracle.run_trace(np.full((1, T), s, dtype=np.uint32), pool, 0, want_ok=False).stats
        row["oracle_failed"] = ref["n_malloc_fail"]
        if "error" not in row["ours"] and "error" not in row["cuda"]:
            row["speedup_block256"] = row["ours"]["allocs_per_s_block256"] / row["cuda"]["allocs_per_s_block256"]
            row["speedup_avg"] = row["ours"]["allocs_per_s_avg_time"] / row["cuda"]["allocs_per_s_avg_time"]
        rows.append(row)
        o, c = row["ours"], row["cuda"]
        print(f"{s:>7d} B  T={T:>8d}  ours {o.get('allocs_per_s_block256', 0):.3e}/s fail {o.get('failed_block256')}"
              f" (oracle {row['oracle_failed']})  cuda {c.get('allocs_per_s_block256', 0):.3e}/s fail "
              f"{c.get('failed_block256')}  x{row.get('speedup_block256', float('nan')):.1f}"
              f"  avg-blocks x{row.get('speedup_avg', float('nan')):.1f}", flush=True)
    sp = [r["speedup_block256"] for r in rows if "speedup_block256" in r]
    spa = [r["speedup_avg"] for r in rows if "speedup_avg" in r]
    out = {"experiment": "Fig. 7 (P:L1508-1698): one malloc per thread, pool exhausted",
           "blocks": blocks_of(a.all_blocks), "rows": rows,
           "mean_speedup_block256": float(np.mean(sp)) if sp else None,
           "mean_speedup_avg_blocks": float(np.mean(spa)) if spa else None,
           "paper_context": "16.56x average over CUDA 9 malloc on GV100 (Titan V), quoted as context only"}
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)
    print(json.dumps({k: out[k] for k in ("mean_speedup_block256", "mean_speedup_avg_blocks")}))
    return 0


if __name__ == "__main__":
    sys.exit(main())
