"""Run d4_small in correctness mode and print the first overlapping pair of blocks."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle, tracegen
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness
torch.cuda.set_device(0)
kmin = int(sys.argv[1]) if len(sys.argv) > 1 else 3
t = tracegen.Trace("x", tracegen.mixed_sizes(tracegen.BASE_SEED + 40, 3, 8192, kmin, 15), 1, 256 << 20, 0)
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
            print("  tid", a[2], "size", a[3], "cls", cls(a[3]), "pages", hex(a[0] >> 12), hex(a[1] >> 12), "| tid", b[2], "size", b[3],
                  "cls", cls(b[3]), "pages", hex(b[0] >> 12), hex(b[1] >> 12), "| warp/lane", a[2] // 32, a[2] % 32, b[2] // 32, b[2] % 32)
            # same-class group mates of a in its warp
            w = a[2] // 32
            mates = [(tt % 32, int(log[2 * (r * T + tt)]['off']) >> 12, cls(int(log[2 * (r * T + tt)]['size'])))
                     for tt in range(w * 32, w * 32 + 32) if cls(int(log[2 * (r * T + tt)]['size'])) == cls(a[3])]
            print("     warp", w, "group (lane, page, cls):", mates)
        break
