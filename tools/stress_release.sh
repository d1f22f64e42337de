#!/bin/bash
# GPU call: release-build liveness stress of the timed kernel (reps per run, watchdog per run).
mkdir -p gpurun_out; : > gpurun_out/stress_rel.log
for occ in ${OCCS:-4 8}; do for sz in ${SIZES:-4096 8192 16}; do for i in $(seq ${RUNS:-2}); do
  echo "== occ $occ size $sz run $i" >> gpurun_out/stress_rel.log
  GA_TIMED_OCC=$occ timeout 150 python tools/profile_trace.py --workload d3 --size $sz --reps ${REPS:-1500} 2>&1 | tail -2 >> gpurun_out/stress_rel.log
done; done; done
