#!/bin/bash
# GPU call: tools/frag_ab.py (d4 ms + fragmentation vs the oracle) for every built variant,
# at the pressure and overcommit levels.
mkdir -p gpurun_out; : > gpurun_out/frag_ab.log
for lib in paper_conf_ppopp_geladog19_b200/variants/libga_*.so; do
  for lv in ${LEVELS:-pressure overcommit}; do
    echo "== $(basename $lib .so) $lv" >> gpurun_out/frag_ab.log
    GA_LIB=$PWD/$lib timeout 300 python tools/frag_ab.py $lv >> gpurun_out/frag_ab.log 2>&1
  done
done
