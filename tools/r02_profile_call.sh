#!/bin/bash
# Round-2 profiling call (the files tools/write_profiles_r02.sh turns into profiles/):
# full bench line, its launch list, ncu --set full of the d4 and d3-16 timed kernels,
# and the per-scope ncu metrics of the collective calls (f4).
mkdir -p gpurun_out
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv \
  python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d4_timed \
  python tools/profile_trace.py --reps 2 > gpurun_out/ncu_d4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d3_16_timed \
  python tools/profile_trace.py --workload d3 --size 16 --reps 2 > gpurun_out/ncu_d3.log 2>&1
SCOPES="0 1 2" bash tools/r02_coll_ncu.sh
tail -3 gpurun_out/bench_full.err
