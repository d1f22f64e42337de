"""Correctness-mode run (log) of a TBuddy/bin mixed trace, guarded by a thread timeout;
prints the first overlapping pairs with warp / lane / class."""
import os, sys, threading
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tracegen
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness
torch.cuda.set_device(0)
kmin = int(sys.argv[1]) if len(sys.argv) > 1 else 3
R = 2
t = tracegen.Trace("x", tracegen.mixed_sizes(tracegen.BASE_SEED + 40, R, 8192, kmin, 15), 1, 256 << 20, 0)
res = {}
def go():
    heap = GpuHeap(t.heap_bytes)
    res["run"] = run_correctness(heap, t.sizes, 1, log=True, tag=True, reserved=False)
th = threading.Thread(target=go, daemon=True); th.start(); th.join(60)
if "run" not in res:
    print("hung"); os._exit(0)
run = res["run"]; log = run.log; T = t.T
print("counts", run.counts)
def blen(n):
    c = 16
    while c < n: c <<= 1
    return max(c, 4096) if c > 2048 else c
for r in range(R):
    iv = []
    for tid in range(T):
        x = log[2 * (r * T + tid)]
        if x['size'] and x['off'] != (1 << 64) - 1:
            iv.append((int(x['off']), int(x['off']) + blen(int(x['size'])), tid, int(x['size'])))
    iv.sort()
    bad = [(a, b) for a, b in zip(iv, iv[1:]) if b[0] < a[1]]
    print("round", r, "blocks", len(iv), "overlaps", len(bad))
    for a, b in bad[:8]:
        print(f"  A tid {a[2]:5d} (w{a[2]//32} l{a[2]%32}) len {a[1]-a[0]:6d} pages {a[0]>>12}-{(a[1]>>12)-1} | "
              f"B tid {b[2]:5d} (w{b[2]//32} l{b[2]%32}) len {b[1]-b[0]:6d} pages {b[0]>>12}-{(b[1]>>12)-1}")
    if bad: break
os._exit(0)
