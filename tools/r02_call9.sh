#!/bin/bash
mkdir -p gpurun_out
REPS=10 bash tools/ab_reps.sh
for sc in 1; do for w in "--workload d4"; do
  r=$(timeout 120 python tools/profile_trace.py $w --scope $sc --reps 10 2>&1 | grep "^rep" | tail -n +3 | awk '{printf "%s ", $3}')
  echo "scope$sc | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab_reps.log
done; done
timeout 120 python tools/profile_trace.py --workload d4 --reps 8 --stats > gpurun_out/d4_stats.log 2>&1
NO_BENCH=1 PER_TEST=150 bash tools/gpu_tests.sh tests/test_gpu_collective.py
cat gpurun_out/ab_reps.log
