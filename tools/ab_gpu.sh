#!/bin/bash
# GPU call: time every built variant (paper_conf_ppopp_geladog19_b200/variants/*.so) on
# d4 (cold) and d3 16 B / 256 B / 4 KiB with the timed kernel (median of reps).
# A variant named *_occN runs with GA_TIMED_OCC=N.
mkdir -p gpurun_out
: > gpurun_out/ab.log
for lib in paper_conf_ppopp_geladog19_b200/variants/libga_*.so; do
  n=$(basename $lib .so)
  occ=$(echo $n | sed -n 's/.*_occ\([0-9]\).*/\1/p')
  for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256" "--workload d3 --size 4096" ${EXTRA_W}; do
    r=$(GA_TIMED_OCC=${occ:-4} GA_LIB=$PWD/$lib timeout 120 python tools/profile_trace.py $w --reps ${REPS:-8} 2>&1 | grep "^rep" | tail -n +3 | awk '{print $3}' | sort -n | awk '{a[NR]=$1} END{print a[int((NR+1)/2)]}')
    echo "$n | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab.log
  done
done
