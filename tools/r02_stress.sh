#!/bin/bash
# Long liveness stress on the final build: 1,000 cold-heap reps of d4 (warp
# and block scope) and of d3 16 B / 4 KiB / 8 KiB, each run under a watchdog.
mkdir -p gpurun_out; : > gpurun_out/stress.log
for sc in 0 1; do for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 4096" "--workload d3 --size 8192"; do
  s=$(date +%s)
  timeout 600 python tools/profile_trace.py $w --scope $sc --reps ${SREPS:-1000} > gpurun_out/stress_tmp.log 2>&1
  rc=$?
  n=$(grep -c "^rep" gpurun_out/stress_tmp.log)
  echo "scope $sc $w: rc=$rc reps=$n $(( $(date +%s)-s )) s; slowest: $(grep '^rep' gpurun_out/stress_tmp.log | tail -n +2 | awk '{print $3}' | sort -n | tail -1) ms; $(tail -1 gpurun_out/stress_tmp.log)" >> gpurun_out/stress.log
done; done
cat gpurun_out/stress.log
