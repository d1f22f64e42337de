#!/bin/bash
# Round-2 measurement call: L2-atomic peak (+ncu), d2 matrix (+ncu), full bench.
mkdir -p gpurun_out
M=lts__t_requests_op_atom.sum,lts__t_requests_op_red.sum,gpu__time_duration.sum
timeout 300 python tools/l2_peak.py > gpurun_out/l2_live.json
timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/l2_ncu.csv python tools/l2_peak.py --reps 0 > /dev/null 2>&1
timeout 900 python tools/d2_matrix.py > gpurun_out/d2.json
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/d2_ncu.csv -k regex:k_bsem python tools/d2_matrix.py --ncu > gpurun_out/d2_ncu_cfgs.json 2>/dev/null
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
ls -la gpurun_out; tail -c 600 gpurun_out/bench_full.json
