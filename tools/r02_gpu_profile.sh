#!/bin/bash
# GPU call: occupancy sweep of the timed kernel (d4, d3 16 B), the bench launch
# list, and ncu --set full captures of the d4 / d3 timed kernels.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for occ in 2 4 5 6 8; do
  echo "== occ $occ d4" >> gpurun_out/occ.log
  GA_TIMED_OCC=$occ timeout 120 python tools/profile_trace.py --reps 5 >> gpurun_out/occ.log 2>&1
  echo "== occ $occ d3-16" >> gpurun_out/occ.log
  GA_TIMED_OCC=$occ timeout 120 python tools/profile_trace.py --workload d3 --size 16 --reps 5 >> gpurun_out/occ.log 2>&1
  echo "== occ $occ d3-4096" >> gpurun_out/occ.log
  GA_TIMED_OCC=$occ timeout 120 python tools/profile_trace.py --workload d3 --size 4096 --reps 5 >> gpurun_out/occ.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv \
  python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d4_timed \
  python tools/profile_trace.py --reps 2 > gpurun_out/ncu_d4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d3_16_timed \
  python tools/profile_trace.py --workload d3 --size 16 --reps 2 > gpurun_out/ncu_d3.log 2>&1
