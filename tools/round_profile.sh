#!/bin/bash
# GPU call for the committed evidence: gpu tests, smoke, the bench line, the
# bench launch list (ncu, serialised) and ncu --set full captures of the timed
# kernel on d4 and d3 16 B.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1; echo bench_rc=$? >> gpurun_out/bench.log
[ -n "$SKIP_NCU" ] && exit 0
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv \
  python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d4_timed \
  python tools/profile_trace.py --reps 2 > gpurun_out/ncu_d4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d3_16_timed \
  python tools/profile_trace.py --workload d3 --size 16 --reps 2 > gpurun_out/ncu_d3.log 2>&1
