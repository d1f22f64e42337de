"""Run d4_small in correctness mode and print the first overlapping pair of blocks."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle, tracegen
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness
torch.cuda.set_device(0)
t = tracegen.d4_small(T=8192, R=8, heap_bytes=256 << 20)
heap = GpuHeap(t.heap_bytes)
run = run_correctness(heap, t.sizes, t.D)
err, cs = oracle.check_log(run.log, t.R, t.T, t.D, t.heap_bytes)
print("checker", err, cs, run.counts)
log = run.log
def cls(n):
    c = 16
    while c < n: c <<= 1
    return c
T = t.T
for r in range(t.R):
    m = log[2 * (r * T + np.arange(T))]
    held = {}
    # live set after round r: the mallocs of round r (D=1: previous blocks freed in this round)
    iv = [(int(x['off']), int(x['off']) + max(cls(int(x['size'])), 4096 if cls(int(x['size'])) > 2048 else 0), tid, int(x['size']))
          for tid, x in enumerate(m) if x['off'] != (1 << 64) - 1 and x['size']]
    iv.sort()
    bad = [(a, b) for a, b in zip(iv, iv[1:]) if b[0] < a[1]]
    if bad:
        print("round", r, "overlaps:", len(bad))
        for a, b in bad[:6]:
            print("  tid", a[2], "size", a[3], "off", hex(a[0]), "| tid", b[2], "size", b[3], "off", hex(b[0]),
                  "| warps", a[2] // 32, b[2] // 32)
        break
