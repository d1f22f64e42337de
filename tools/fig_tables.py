"""Markdown tables from the Fig. 7 / Fig. 5 JSONs (tools/fig7.py, tools/fig5.py)."""
import json
import sys

import numpy as np


def fig7(path):
    d = json.load(open(path))
    print(f"blocks: {d['blocks']}\n")
    print("| size | threads | ours (allocs/s) | fails (oracle) | CUDA malloc | CUDA fails | speedup (block 256) | speedup (avg over blocks) |")
    print("|---|---|---|---|---|---|---|---|")
    sp, spa = [], []
    for r in d["rows"]:
        o, c = r["ours"], r["cuda"]
        if "error" in o or "error" in c:
            print(f"| {r['size']} B | | {o.get('error', '')[:40]} | | {c.get('error', '')[:40]} | | | |")
            continue
        s256, sav = r.get("speedup_block256"), r.get("speedup_avg")
        sp.append(s256); spa.append(sav)
        print(f"| {r['size']} B | {o['threads']:,} | {o['allocs_per_s_block256']:.3g} | {o['failed_block256']:,} ({r['oracle_failed']:,}) "
              f"| {c['allocs_per_s_block256']:.3g} | {c['failed_block256']:,} | {s256:.1f}x | {sav:.1f}x |")
    print(f"\ngeomean speedup block 256: {np.exp(np.mean(np.log(sp))):.1f}x, avg over blocks: {np.exp(np.mean(np.log(spa))):.1f}x; "
          f"arithmetic means {np.mean(sp):.1f}x / {np.mean(spa):.1f}x")


def fig5(path):
    d = json.load(open(path))
    names = [k for k in d["rows"][0] if k != "threads"]
    print(f"blocks: {d['blocks']}\n")
    print("| threads | " + " | ".join(f"{n} (avg over blocks)" for n in names) + " |")
    print("|---|" + "---|" * len(names))
    for r in d["rows"]:
        print(f"| {r['threads']:,} | " + " | ".join(f"{r[n]['allocs_per_s_avg_time']:.3g}{'' if r[n]['invariants_ok'] else ' (!)'}" for n in names) + " |")


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(f"\n### {p}\n")
        (fig5 if "fig5" in p else fig7)(p)
