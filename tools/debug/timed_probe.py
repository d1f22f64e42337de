"""Malloc-then-free of mixed 1 B - 256 KiB sizes in ONE kernel (the timed kernel,
D = 0), the pattern of tests/test_gpu_edge.py's free pass, under a watchdog."""
import os, sys, threading, time
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_timed
torch.cuda.set_device(0)
T = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
reps = int(os.environ.get("REPS", "20"))
heap = GpuHeap(512 << 20)
done = []
def work():
    for rep in range(reps):
        rng = np.random.default_rng(T + rep)
        sizes = ((1 << rng.integers(0, 18, T)) + rng.integers(0, 7, T)).astype(np.uint32).reshape(1, T)
        d = torch.from_numpy(sizes.view(np.int32)).cuda()
        c = torch.zeros(8, dtype=torch.int64, device="cuda")
        heap.reset()
        run_timed(heap, d, 1, T, 0, c)
        torch.cuda.synchronize()
        print("rep", rep, c.cpu().numpy()[:3], flush=True)
    done.append(1)
threading.Thread(target=work, daemon=True).start()
for sec in range(int(os.environ.get("PROBE_S", "30"))):
    time.sleep(1)
    if done:
        print("finished"); break
else:
    print("HANG after", sec + 1, "s")
sys.stdout.flush()
os._exit(0)
