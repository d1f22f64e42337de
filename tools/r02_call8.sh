#!/bin/bash
mkdir -p gpurun_out
bash tools/ab_reps.sh
for sc in 1 2; do for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256"; do
  r=$(timeout 120 python tools/profile_trace.py $w --scope $sc --reps 8 2>&1 | grep "^rep" | tail -n +3 | awk '{printf "%s ", $3}')
  echo "scope$sc | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab_reps.log
done; done
GA_LIB=$PWD/paper_conf_ppopp_geladog19_b200/variants/libga_def.so timeout 120 python tools/profile_trace.py --workload d4 --reps 6 --stats > gpurun_out/d4_stats.log 2>&1
bash tools/iter_stats.sh
NO_BENCH=1 PER_TEST=150 bash tools/gpu_tests.sh tests/test_gpu_collective.py tests/test_gpu_parity.py tests/test_gpu_edge.py tests/test_gpu_scale.py
cat gpurun_out/ab_reps.log
