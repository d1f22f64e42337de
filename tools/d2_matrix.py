"""d2, the bulk-semaphore microbenchmark over its whole matrix (SURVEY 8(d),
BASELINE configs[1]; "other batch sizes are analogous").

Full grid (148 x 8 x 256 threads), each thread `iters` x {wait(k); signal(k)}:
k in {1, 2, 4, 8, 16, 32, per-lane random 1..32}, B in {32, 512, 4096},
1 global or 148 per-SM semaphores, variants (i) warp-aggregated bulk,
(ii) per-thread bulk, (iii) per-thread counting (k = 1), (iv) plain per-thread
atomics.  Every run's accounting is checked (quiescent C = units produced,
D = 0).  With --ncu the same launches are replayed under ncu by the caller and
--ncu-csv attaches L2 atom/red requests per wait+signal pair to each entry.

usage (GPU box): python tools/d2_matrix.py > gpurun_out/d2.json
                 ncu --metrics lts__t_requests_op_atom.sum,lts__t_requests_op_red.sum --csv \
                     --log-file gpurun_out/d2_ncu.csv -k regex:k_bsem$ python tools/d2_matrix.py --ncu
                 (its stdout -> gpurun_out/d2_ncu_cfgs.json)
here:            python tools/d2_matrix.py --merge gpurun_out/d2.json --ncu-cfgs gpurun_out/d2_ncu_cfgs.json \
                     --ncu-csv gpurun_out/d2_ncu.csv
"""
import argparse
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
GRID, BLOCK = 148 * 8, 256
VARIANTS = {0: "warp_bulk", 1: "thread_bulk", 2: "thread_counting", 3: "plain_atomics"}


def configs(ncu):
    for n_sems in (1, 148):
        for B in (32, 512, 4096):
            for k in (1, 2, 4, 8, 16, 32, 0):
                for v in VARIANTS:
                    if v == 2 and k != 1:
                        continue
                    if ncu and (B != 512 or k not in (1, 32, 0)):
                        continue
                    yield v, k, B, n_sems


def run(ncu):
    import torch
    import paper_conf_ppopp_geladog19_b200 as ga
    import tracegen
    torch.cuda.set_device(0)
    s = torch.cuda.current_stream()
    sems = torch.zeros(148 * 4 + 8, dtype=torch.int64, device="cuda")
    out_t = torch.zeros(8, dtype=torch.int64, device="cuda")
    res = []
    def launch(cfg):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        ga.ga_bsem_bench(s.cuda_stream, cfg, sems.data_ptr(), out_t.data_ptr())
        e1.record(s)
        e1.synchronize()
        return e0.elapsed_time(e1) / 1e3

    for v, k, B, n_sems in configs(ncu):
        cfg = ga.BsemCfg(variant=v, k=k, B=B, n_sems=n_sems, iters=1, acquire_only=0, grid=GRID, block=BLOCK,
                         seed=tracegen.BASE_SEED + 2)
        probe = launch(cfg) if not ncu else None                # size the run to ~50 ms, 1..32 iterations
        iters = 2 if ncu else max(1, min(32, int(0.05 / max(probe, 1e-6))))
        cfg.iters = iters
        best = None
        for rep in range(1 if ncu else 3):
            t = launch(cfg)
            best = t if best is None else min(best, t)
        o = out_t.cpu().numpy()
        pairs = GRID * BLOCK * iters
        res.append({"variant": VARIANTS[v], "k": k or "rand", "B": B, "sems": n_sems, "iters": iters,
                    "pairs": pairs, "seconds": best, "G_pairs_s": pairs / best / 1e9,
                    "units_granted": int(o[0]), "batches": int(o[2]),
                    "accounting_ok": bool(o[4] == o[3] and o[5] == 0)})
    return res


def merge(res_json, ncu_cfgs_json, ncu_csv):
    """Attach ncu's L2 atom + red requests per wait+signal pair (from the --ncu
    run, whose launches follow its printed config list) to the timing entries."""
    res = json.load(open(res_json))
    cfgs = json.load(open(ncu_cfgs_json))
    rows = list(csv.DictReader(l for l in open(ncu_csv) if not l.startswith("==")))
    per = {}
    for r in rows:
        name = r.get("Kernel Name", "")
        if "k_bsem" not in name or "final" in name or "init" in name:
            continue
        per.setdefault(int(r["ID"]), {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    launches = [per[k] for k in sorted(per)]
    assert len(launches) == len(cfgs), (len(launches), len(cfgs))
    key = lambda e: (e["variant"], str(e["k"]), e["B"], e["sems"])  # noqa: E731
    by = {key(e): e for e in res}
    for c, m in zip(cfgs, launches):
        req = m.get("lts__t_requests_op_atom.sum", 0) + m.get("lts__t_requests_op_red.sum", 0)
        by[key(c)]["ncu_l2_atom_red_per_pair"] = round(req / c["pairs"], 4)
    return res


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--ncu", action="store_true")
    ap.add_argument("--merge")
    ap.add_argument("--ncu-cfgs")
    ap.add_argument("--ncu-csv")
    a = ap.parse_args()
    if a.merge:
        out = merge(a.merge, a.ncu_cfgs, a.ncu_csv)
        json.dump(out, open(os.path.join(ROOT, "profiles", "r02_d2_matrix.json"), "w"), indent=0)
        print(len(out), "entries")
    else:
        print(json.dumps(run(a.ncu)))
