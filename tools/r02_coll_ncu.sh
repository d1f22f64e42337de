#!/bin/bash
# f4 evidence: L2 atomic / reduction requests, instructions and time of the
# timed kernel per call scope (0 warp, 1 block, 2/4 cluster) on d3 16 B,
# d3 256 B and d4 (one launch each after a warm-up launch).
mkdir -p gpurun_out
M=lts__t_requests_srcunit_tex_op_atom_dot_alu.sum,lts__t_requests_srcunit_tex_op_atom_dot_cas.sum,lts__t_requests_srcunit_tex_op_red.sum,gpu__time_duration.sum,smsp__inst_executed.sum,smsp__thread_inst_executed_per_inst_executed.ratio,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
for sc in ${SCOPES:-0 1 2 4}; do
  for w in "d4:--workload d4" "d3_16:--workload d3 --size 16" "d3_256:--workload d3 --size 256"; do
    name=${w%%:*}; args=${w#*:}
    timeout 600 ncu --metrics $M --clock-control none -k regex:k_timed -s 1 -c 1 --csv \
      --log-file gpurun_out/coll_ncu_s${sc}_${name}.csv python tools/profile_trace.py $args --scope $sc --reps 2 \
      > gpurun_out/coll_ncu_s${sc}_${name}.log 2>&1
    echo "scope $sc $name rc=$?"
  done
done
