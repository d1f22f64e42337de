#!/bin/bash
mkdir -p gpurun_out; : > gpurun_out/call12.log
s=$(date +%s); timeout 300 python bench.py --steps 10 --warmup 3 --no-extras > gpurun_out/bench_short.json 2>&1; echo "bench no-extras rc=$? $(( $(date +%s)-s ))s" >> gpurun_out/call12.log
for lv in fit exhaust overcommit; do
  s=$(date +%s); timeout 120 python tools/profile_trace.py --level $lv --reps 3 --stats >> gpurun_out/call12.log 2>&1; echo "level $lv rc=$? $(( $(date +%s)-s ))s" >> gpurun_out/call12.log
done
s=$(date +%s); timeout 600 python -m pytest tests/test_gpu_scale.py -m gpu -q -x -p no:cacheprovider --timeout 150 >> gpurun_out/call12.log 2>&1; echo "scale rc=$? $(( $(date +%s)-s ))s" >> gpurun_out/call12.log
cat gpurun_out/call12.log | tail -40
