"""Build tuning variants of libga.so (compile-time switches) for A/B timing on the GPU.
usage: build_variants.py name=DEF1,DEF2 name2=DEF3 ...  -> paper_conf_ppopp_geladog19_b200/variants/libga_<name>.so"""
import os
import sys
from concurrent.futures import ThreadPoolExecutor

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_geladog19_b200 import _build  # noqa: E402

out_dir = os.path.join(_build.PKG, "variants")
os.makedirs(out_dir, exist_ok=True)
jobs = []
for arg in sys.argv[1:]:
    name, _, defs = arg.partition("=")
    jobs.append((name, tuple(d for d in defs.split(",") if d)))
with ThreadPoolExecutor(8) as ex:
    for name, path in zip([j[0] for j in jobs],
                          ex.map(lambda j: _build.build(defines=j[1], out=os.path.join(out_dir, f"libga_{j[0]}.so")), jobs)):
        print(name, path)
