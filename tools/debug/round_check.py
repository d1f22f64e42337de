"""d4_small round by round; after each round check the GPU snapshot with the oracle's invariants."""
import os, sys, threading, time
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tracegen
from oracle import snapshot as S
from paper_conf_ppopp_geladog19_b200 import ga_trace_phase, GA_TRACE_TAG
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap
torch.cuda.set_device(0)
T = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
kmin = int(sys.argv[2]) if len(sys.argv) > 2 else 3
t = tracegen.Trace("x", tracegen.mixed_sizes(tracegen.BASE_SEED + 40, 8, T, kmin, 15), 1, 256 << 20, 0)
heap = GpuHeap(t.heap_bytes)
d = torch.from_numpy(t.sizes.view(np.int32)).cuda()
held = torch.empty(2 * T, dtype=torch.int64, device="cuda"); held[0::2] = -1; held[1::2] = 0
c = torch.zeros(8, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream
def go():
    for r in range(t.R + 1):
        ga_trace_phase(heap.h, s, d.data_ptr(), t.R, T, 1, r, 0, held.data_ptr(), 0, c.data_ptr(), GA_TRACE_TAG, 256)
        torch.cuda.synchronize()
        snap = S.parse(heap.snapshot())
        errs = S.check(snap)
        print("round", r, "counts", c.cpu().numpy()[:4], "errors", errs[:4], flush=True)
        if errs:
            # dump semaphore vs bitmap per level
            for n, bits in enumerate(snap.level_bits):
                if snap.tree_C[n] != bits.sum() or snap.tree_D[n]:
                    print("  level", n, "C", snap.tree_C[n], "avail", int(bits.sum()), "D", snap.tree_D[n], flush=True)
            break
th = threading.Thread(target=go, daemon=True); th.start(); th.join(60)
print("alive" if th.is_alive() else "done", flush=True)
os._exit(0)
