import os, sys, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tracegen
from paper_conf_ppopp_geladog19_b200.runner import GpuHeap, run_correctness
torch.cuda.set_device(0)
T = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
sizes = np.full((1, T), int(sys.argv[2]) if len(sys.argv) > 2 else 16, dtype=np.uint32)
heap = GpuHeap(1 << 20 if T <= 1024 else 64 << 20)
print("created", flush=True)
run = run_correctness(heap, sizes, 0, log=False)
print(run.counts, heap.stats(), flush=True)
