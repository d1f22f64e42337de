"""Per-round diagnostics of a churn trace: GPU (correctness mode) vs oracle.
Prints reserved / live / failures / reclamation state per round.  Not a bench."""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tracegen  # noqa: E402
from paper_conf_ppopp_geladog19_b200 import GA_TRACE_TAG, ga_trace_phase  # noqa: E402
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--T", type=int, default=8192)
ap.add_argument("--R", type=int, default=8)
ap.add_argument("--heap-mib", type=int, default=96)
a = ap.parse_args()
t = tracegen.d4_small(T=a.T, R=a.R, heap_bytes=a.heap_mib << 20)
torch.cuda.set_device(0)
heap = GpuHeap(t.heap_bytes)
d_sizes = torch.from_numpy(t.sizes.view(np.int32)).cuda()
held = torch.empty(2 * t.T, dtype=torch.int64, device="cuda")
held[0::2] = -1
held[1::2] = 0
counts = torch.zeros(8, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream
print("round  gpu_reserved_MiB  gpu_live_MiB  gpu_fail  bin_grow chunk_grow bin_recl chunk_recl pending fallback")
prev_fail = 0
for r in range(t.R + 1):
    ga_trace_phase(heap.h, s, d_sizes.data_ptr(), t.R, t.T, 1, r, 0, held.data_ptr(), 0, counts.data_ptr(),
                   GA_TRACE_TAG, 256)
    torch.cuda.synchronize()
    st = heap.stats()
    c = counts.cpu().numpy()
    live = int(held[1::2].sum().item())
    print(f"{r:5d} {st['reserved_bytes'] / 2**20:17.1f} {live / 2**20:13.1f} {int(c[1]) - prev_fail:9d} "
          f"{st['n_bin_grow']:8d} {st['n_chunk_grow']:10d} {st['n_bin_reclaim']:8d} {st['n_chunk_reclaim']:10d} "
          f"{st['n_pending_reclaim']:7d} {st['n_fallback']:8d}")
    prev_fail = int(c[1])
print("tag errors", int(counts[3].item()))
ref = oracle.run_trace(t.sizes, t.heap_bytes, t.D)
print("oracle:", {k: ref.stats[k] for k in ("n_malloc_fail", "peak_live_bytes", "peak_reserved_bytes",
                                             "n_bin_grow", "n_chunk_grow")})
# per-round oracle failures
for r in range(1, t.R + 1):
    rr = oracle.run_trace(t.sizes[:r], t.heap_bytes, t.D)
    print(f"oracle rounds<= {r}: fails {rr.stats['n_malloc_fail']} peak_res_MiB {rr.stats['peak_reserved_bytes']/2**20:.1f}"
          f" peak_live_MiB {rr.stats['peak_live_bytes']/2**20:.1f}")
