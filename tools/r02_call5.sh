#!/bin/bash
mkdir -p gpurun_out
REPS=6 bash tools/ab_gpu.sh
for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256"; do
  echo "== cnt $w" >> gpurun_out/ab.log
  GA_LIB=$PWD/paper_conf_ppopp_geladog19_b200/variants/libga_cnt.so timeout 120 python tools/profile_trace.py $w --reps 1 2>&1 | tail -2 >> gpurun_out/ab.log
done
for sc in 1 2; do
  for w in "--workload d4" "--workload d3 --size 16"; do
    r=$(timeout 120 python tools/profile_trace.py $w --scope $sc --reps 6 2>&1 | grep "^rep" | tail -n +3 | awk '{print $3}' | sort -n | awk '{a[NR]=$1} END{print a[int((NR+1)/2)]}')
    echo "default_scope$sc | $w | ${r:-HANG/FAIL}" >> gpurun_out/ab.log
  done
done
cat gpurun_out/ab.log
T=40 LINES_OUT=120 bash tools/debug/gdb_run.sh gdb_coll python tools/debug/coll_probe.py 256 16461 1 0 2 > /dev/null 2>&1
