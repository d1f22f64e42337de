#!/bin/bash
# GA_COUNT_ITERS build: lockstep calls and warp iterations per workload
# (d3 per class, d4 sub-ranges of octaves)
mkdir -p gpurun_out; : > gpurun_out/iter_stats.log
L=$PWD/paper_conf_ppopp_geladog19_b200/variants/libga_cnt.so
for w in "--workload d4" "--workload d4 --kmin 3 --kmax 10" "--workload d4 --kmin 11 --kmax 15" "--workload d4 --kmin 3 --kmax 6" \
         "--workload d3 --size 16" "--workload d3 --size 64" "--workload d3 --size 256" "--workload d3 --size 1024" \
         "--workload d3 --size 2048" "--workload d3 --size 4096" "--workload d3 --size 16384" "--workload d3 --size 65536"; do
  r=$(GA_LIB=$L timeout 120 python tools/profile_trace.py $w --reps 1 2>&1 | tail -2 | tr '\n' ' ')
  echo "$w | $r" >> gpurun_out/iter_stats.log
done
cat gpurun_out/iter_stats.log
