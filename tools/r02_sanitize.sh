#!/bin/bash
# compute-sanitizer memcheck / synccheck / racecheck on reduced traces at every
# call scope; each run's summary lines (or its last lines on failure) kept.
mkdir -p gpurun_out; : > gpurun_out/sanitize.log
CS=/usr/local/cuda/bin/compute-sanitizer
for sc in 0 1 2; do
  for w in "--workload d3 --size 4096" "--workload d4" "--workload d3 --size 16"; do
    for tool in memcheck synccheck racecheck; do
      echo "== $tool scope $sc $w" >> gpurun_out/sanitize.log
      timeout 900 $CS --tool $tool --print-limit 10 python tools/profile_trace.py $w --scope $sc --rounds 2 --reps 1 --threads 8192 \
        > gpurun_out/san_tmp.log 2>&1
      echo "rc=$?" >> gpurun_out/sanitize.log
      grep -E "SUMMARY|^rep |Error|error|Hazard|hazard" gpurun_out/san_tmp.log | head -12 >> gpurun_out/sanitize.log
      grep -qE "SUMMARY" gpurun_out/san_tmp.log || tail -5 gpurun_out/san_tmp.log >> gpurun_out/sanitize.log
    done
  done
done
cat gpurun_out/sanitize.log | head -150
