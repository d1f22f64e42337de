"""A/B helper: d4 pressure timed-kernel ms (heap reset between reps) and the
correctness-mode fragmentation against the oracle's, for the libga.so named by
GA_LIB (a tuning variant) or the default build.  Not a bench number."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tracegen  # noqa: E402
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness, run_timed  # noqa: E402

level = sys.argv[1] if len(sys.argv) > 1 else "pressure"
t = tracegen.d4_mixed(level, R=16)
torch.cuda.set_device(0)
heap = GpuHeap(t.heap_bytes)
d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
c = torch.zeros(8, dtype=torch.int64, device="cuda")
ms = []
for i in range(4):
    heap.reset()
    c.zero_()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    run_timed(heap, d, t.R, t.T, t.D, c)
    e.record()
    e.synchronize()
    ms.append(s.elapsed_time(e))
fails = int(c[1].item())
warm = []
for i in range(6):                                   # steady state, as bench.py times it (no reset)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    run_timed(heap, d, t.R, t.T, t.D, c)
    e.record()
    e.synchronize()
    warm.append(s.elapsed_time(e))
warm = sorted(warm[2:])
heap.reset()
run = run_correctness(heap, t.sizes, t.D, log=False, tag=False, reserved=True)
ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
fg = run.peak_reserved_bytes / run.peak_live_bytes
fo = ref.stats["peak_reserved_bytes"] / ref.stats["peak_live_bytes"]
print(f"{os.environ.get('GA_LIB', 'default')}: {level} cold ms {[round(x, 2) for x in sorted(ms)[1:]]} warm ms {[round(x, 2) for x in warm]} timed_fails {fails} "
      f"frag gpu {fg:.4f} oracle {fo:.4f} ratio {fg / fo:.4f} reserved {run.peak_reserved_bytes / 2**30:.3f} GiB "
      f"fails {run.counts['n_fail']}", flush=True)
