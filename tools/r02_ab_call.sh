#!/bin/bash
# Round-2 A/B call: variant timings (tools/ab_gpu.sh), the collective-scope
# timings of the default build, then the GPU parity tests of the default build.
mkdir -p gpurun_out
REPS=${REPS:-6} bash tools/ab_gpu.sh
for sc in ${SCOPES:-1 2 4}; do
  for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256"; do
    r=$(timeout 120 python tools/profile_trace.py $w --scope $sc --reps 6 2>&1 | grep "^rep" | tail -n +3 | awk '{print $3}' | sort -n | awk '{a[NR]=$1} END{print a[int((NR+1)/2)]}')
    echo "default_scope$sc | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab.log
  done
done
cat gpurun_out/ab.log
NO_BENCH=1 PER_TEST=240 bash tools/gpu_tests.sh ${TESTS}
