#!/bin/bash
# every rep time (ms) of each variant on d4 / d3 16 B / d3 256 B (first 2 reps warm-up)
mkdir -p gpurun_out; : > gpurun_out/ab_reps.log
for lib in paper_conf_ppopp_geladog19_b200/variants/libga_*.so; do
  n=$(basename $lib .so); occ=$(echo $n | sed -n 's/.*_occ\([0-9]\).*/\1/p')
  for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256" ${EXTRA_W}; do
    r=$(GA_TIMED_OCC=${occ:-4} GA_LIB=$PWD/$lib timeout 120 python tools/profile_trace.py $w --reps ${REPS:-8} 2>&1 | grep "^rep" | tail -n +3 | awk '{printf "%s ", $3}')
    echo "$n | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab_reps.log
  done
done
cat gpurun_out/ab_reps.log
