"""the paper's Fig. 6 experiment on one B200.

Doubly-linked-list tag removal under SRCU: T threads, a list of W = T / ratio
elements, every list tag once in the input (writers) and T - W tags that miss
(readers).  Classical RCU (every writer runs a full barrier) against RCU
delegation (conditional barriers), for writer:reader ratios
1:32 .. 1:2048.  Each run is checked against the oracle's outcome
(oracle.rcu.list_removal): every list element removed exactly once, the list
empty, no release while a reader could hold the element.
  python tools/fig6.py [--out profiles/r01_fig6.json]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

THREADS = [4096, 16384, 65536, 131072, 262144]
RATIOS = [32, 128, 512, 2048]


def run(ga, torch, T, W, delegate, reps=2):
    import tracegen
    tags = torch.from_numpy(tracegen.rcu_tags(T, W).view(np.int32)).cuda()
    wsb = ga.ga_rcu_workspace_bytes(W)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    out = torch.zeros(8, dtype=torch.int64, device="cuda")
    st = torch.cuda.current_stream().cuda_stream
    best = None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ga.ga_rcu_list_removal(st, T, W, tags.data_ptr(), ws.data_ptr(), wsb, int(delegate), 256, out.data_ptr())
        e1.record()
        e1.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
    o = [int(x) for x in out.cpu().numpy()]
    ok = o[0] == W and o[1] == W and o[2] == 0 and o[5] == 0 and o[6] == 0 and o[7] == T - W
    return {"seconds": best, "unlinked": o[0], "released": o[1], "violations": o[2], "full_barriers": o[3],
            "delegated": o[4], "double_releases": o[5], "list_len_after": o[6], "readers": o[7], "oracle_ok": ok}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--threads", default=None)
    ap.add_argument("--max-writers", type=int, default=2048)
    a = ap.parse_args()
    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    import oracle.rcu as orcu
    import tracegen
    torch.cuda.set_device(0)
    rows = []
    for T in ([int(x) for x in a.threads.split(",")] if a.threads else THREADS):
        for r in RATIOS:
            W = max(1, T // r)
            if W > a.max_writers:              # classical RCU runs W serial barriers of one traversal each
                print(f"T={T:>7d} 1:{r:<5d} W={W:>6d}  skipped (W > {a.max_writers})", flush=True)
                continue
            removed, live = orcu.list_removal(range(W), tracegen.rcu_tags(T, W).tolist())
            assert sorted(removed) == list(range(W)) and live == []
            cl = run(ga, torch, T, W, False)
            dl = run(ga, torch, T, W, True)
            row = {"threads": T, "ratio": f"1:{r}", "writers": W, "classical": cl, "delegation": dl,
                   "speedup": cl["seconds"] / dl["seconds"]}
            rows.append(row)
            print(f"T={T:>7d} 1:{r:<5d} W={W:>6d}  classical {cl['seconds'] * 1e3:9.2f} ms ({cl['full_barriers']} barriers)"
                  f"  delegation {dl['seconds'] * 1e3:9.2f} ms ({dl['full_barriers']} barriers, {dl['delegated']} delegated)"
                  f"  x{row['speedup']:.2f}  ok {cl['oracle_ok'] and dl['oracle_ok']}", flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"experiment": "Fig. 6 (P:L1404-1478): SRCU list removal, classical vs delegation",
                       "rows": rows}, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
