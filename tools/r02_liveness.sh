#!/bin/bash
# repeated-rep liveness of the timed kernel at warp and block scope (cold heap
# per rep), including d3 64 KiB, whose resident demand exceeds the 4 GiB heap
# at block scope (every thread of a block holds its block until the call ends)
mkdir -p gpurun_out; : > gpurun_out/liveness.log
for sc in 0 1; do for w in "--workload d4" "--workload d3 --size 8192" "--workload d3 --size 65536"; do
  echo "== liveness scope $sc $w (reps ${LREPS:-200})" >> gpurun_out/liveness.log
  s=$(date +%s)
  timeout 400 python tools/profile_trace.py $w --scope $sc --reps ${LREPS:-200} > gpurun_out/live_tmp.log 2>&1
  echo "rc=$? $(( $(date +%s)-s )) s; slowest reps:" >> gpurun_out/liveness.log
  grep "^rep" gpurun_out/live_tmp.log | sort -t: -k2 -n -r | head -2 >> gpurun_out/liveness.log 2>/dev/null
  grep "^rep" gpurun_out/live_tmp.log | sort -k3 -n -r | head -2 >> gpurun_out/liveness.log
  tail -2 gpurun_out/live_tmp.log >> gpurun_out/liveness.log
done; done
cat gpurun_out/liveness.log
