"""Run the timed trace kernel a few times (for ncu captures).  Not a bench number."""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tracegen  # noqa: E402
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_timed  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="d4")
ap.add_argument("--size", type=int, default=16)
ap.add_argument("--rounds", type=int, default=16)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--cuda", action="store_true")
ap.add_argument("--kmin", type=int, default=3)
ap.add_argument("--kmax", type=int, default=15)
ap.add_argument("--threads", type=int, default=0, help="fewer threads than the full grid (sanitizer runs)")
ap.add_argument("--stats", action="store_true", help="heap stats after every rep")
ap.add_argument("--scope", type=int, default=0, help="0 warp calls, 1 block-collective, 2..8 cluster-collective")
ap.add_argument("--warm", action="store_true", help="no heap reset between reps")
ap.add_argument("--level", default="pressure", help="d4 pressure level (fit / pressure / exhaust / overcommit)")
a = ap.parse_args()
if a.workload == "d4":
    t = tracegen.d4_mixed(a.level, R=a.rounds)
    if (a.kmin, a.kmax) != (3, 15):
        t = tracegen.Trace("d4_sub", tracegen.mixed_sizes(t.seed, a.rounds, t.T, a.kmin, a.kmax), 1, t.heap_bytes, t.seed)
else:
    t = tracegen.d3_uniform(a.size, R=a.rounds)
if a.threads:
    t = tracegen.Trace(t.name, np.ascontiguousarray(t.sizes[:, :a.threads]), t.D, t.heap_bytes, t.seed)
torch.cuda.set_device(0)
heap = None if a.cuda else GpuHeap(t.heap_bytes)
if a.cuda:
    import paper_conf_ppopp_geladog19_b200 as ga
    ga.ga_cuda_set_heap_limit(t.heap_bytes)
d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
c = torch.zeros(8, dtype=torch.int64, device="cuda")
for i in range(a.reps):
    if heap is not None and not a.warm:
        heap.reset()                                   # cold heap per rep, as bench.py times it
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    run_timed(heap, d, t.R, t.T, t.D, c, scope=a.scope)
    e.record()
    e.synchronize()
    print(f"rep {i}: {s.elapsed_time(e):.2f} ms, counts {c.cpu().numpy()[:4]}", flush=True)
    if a.stats and heap is not None:
        st = heap.stats()
        print("  ", {k: st[k] for k in ("peak_reserved_bytes", "n_bin_grow", "n_chunk_grow", "n_bin_reclaim", "n_fallback",
                                      "n_waiter_reclaim", "n_fail")}, flush=True)
if heap is not None:
    st = heap.stats()
    print("stats", {k: st[k] for k in ("n_repair_nonfull", "n_repair_summary", "n_fallback", "n_fail")}, flush=True)
