"""Correctness-mode run of a (sub-)mixed trace at full grid, checked by the oracle's log checker."""
import argparse, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle, tracegen
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness, run_timed
ap = argparse.ArgumentParser()
ap.add_argument("--kmin", type=int, default=3); ap.add_argument("--kmax", type=int, default=15)
ap.add_argument("--R", type=int, default=2); ap.add_argument("--T", type=int, default=303104)
ap.add_argument("--heap-gib", type=int, default=4)
a = ap.parse_args()
torch.cuda.set_device(0)
sizes = tracegen.mixed_sizes(tracegen.BASE_SEED + 4, a.R, a.T, a.kmin, a.kmax)
hb = a.heap_gib << 30
heap = GpuHeap(hb)
run = run_correctness(heap, sizes, 1, log=True, tag=True, reserved=True)
print("counts", run.counts, "peak_live", run.peak_live_bytes, "peak_res", run.peak_reserved_bytes)
err, cs = oracle.check_log(run.log, a.R, a.T, 1, hb)
print("checker", err, cs)
heap.reset()
d = torch.from_numpy(sizes.view(np.int32)).cuda()
c = torch.zeros(8, dtype=torch.int64, device="cuda")
run_timed(heap, d, a.R, a.T, 1, c); torch.cuda.synchronize()
print("timed counts", c.cpu().numpy()[:4])
ref = oracle.run_trace(sizes, hb, 1)
print("oracle", {k: ref.stats[k] for k in ("n_malloc", "n_malloc_fail", "n_free", "peak_live_bytes")})
