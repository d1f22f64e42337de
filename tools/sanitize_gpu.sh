#!/bin/bash
# GPU call: compute-sanitizer synccheck / racecheck-free memcheck on reduced traces.
mkdir -p gpurun_out; : > gpurun_out/sanitize.log
for w in "--workload d3 --size 8192" "--workload d3 --size 4096" "--workload d4"; do
  echo "== synccheck $w" >> gpurun_out/sanitize.log
  timeout 600 compute-sanitizer --tool synccheck --print-limit 20 python tools/profile_trace.py $w --rounds 4 --reps 2 --threads 16384 >> gpurun_out/sanitize.log 2>&1
  echo "== memcheck $w" >> gpurun_out/sanitize.log
  timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/profile_trace.py $w --rounds 4 --reps 2 --threads 16384 >> gpurun_out/sanitize.log 2>&1
done
