"""Timed-kernel reps on a warp-uniform trace; after each rep (quiescent) compare
every class semaphore's C with the free slots the snapshot shows.  Finds the
first rep where the accounting drifts.  usage: drift_check.py SIZE [REPS]"""
import os, sys, threading
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tracegen
from oracle import snapshot as S
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_timed
torch.cuda.set_device(0)
size = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 200
t = tracegen.d3_uniform(size, R=16)
heap = GpuHeap(t.heap_bytes)
d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
c = torch.zeros(8, dtype=torch.int64, device="cuda")

def go():
    for r in range(reps):
        run_timed(heap, d, t.R, t.T, t.D, c)
        torch.cuda.synchronize()
        s = S.parse(heap.snapshot())
        free = np.zeros(s.ncls + s.nspan, dtype=np.int64)
        nb = np.zeros(s.ncls + s.nspan, dtype=np.int64)
        for p, bits in s.bins.items():
            k = s.page_class(p)
            free[k] += int((~bits).sum()); nb[k] += 1
        bad = [(k, int(s.cls_C[k]), int(free[k]), int(nb[k]), int(s.cls_absD[k])) for k in range(len(free))
               if s.cls_C[k] != free[k] or s.cls_absD[k]]
        st = heap.stats()
        print(f"rep {r}: drift {bad} bins {nb.tolist()} reclaims {st['n_bin_reclaim']} grows {st['n_bin_grow']} "
              f"fallback {st['n_fallback']} fail {st['n_fail']}", flush=True)
        if bad:
            break
th = threading.Thread(target=go, daemon=True); th.start(); th.join(float(os.environ.get("BUDGET_S", "240")))
print("alive (hung?)" if th.is_alive() else "done", flush=True)
os._exit(0)
