#!/bin/bash
# Round-2 evidence call: compute-sanitizer (memcheck, synccheck, racecheck) on
# reduced traces at every call scope, a repeated-rep liveness run, the ncu
# captures the verdict asked for (CUDA-malloc comparator, d4-exhaust DRAM).
mkdir -p gpurun_out; : > gpurun_out/sanitize.log; : > gpurun_out/liveness.log
for sc in 0 1 2; do
  for w in "--workload d3 --size 4096" "--workload d4" "--workload d3 --size 16"; do
    for tool in memcheck synccheck racecheck; do
      echo "== $tool scope $sc $w" >> gpurun_out/sanitize.log
      timeout 600 compute-sanitizer --tool $tool --print-limit 20 python tools/profile_trace.py $w --scope $sc --rounds 4 --reps 2 --threads 16384 2>&1 \
        | grep -E "ERROR SUMMARY|RACECHECK SUMMARY|========= (Error|Invalid|Race|Barrier)|^rep 1" >> gpurun_out/sanitize.log
    done
  done
done
for sc in 0 1; do for w in "--workload d4" "--workload d3 --size 8192" "--workload d3 --size 65536"; do
  echo "== liveness scope $sc $w" >> gpurun_out/liveness.log
  timeout 300 python tools/profile_trace.py $w --scope $sc --reps ${LREPS:-300} 2>&1 | tail -2 >> gpurun_out/liveness.log
done; done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_requests_srcunit_tex_op_atom_dot_alu.sum,lts__t_requests_srcunit_tex_op_red.sum,smsp__inst_executed.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:k_timed -c 1 --csv --log-file gpurun_out/ncu_cuda_malloc_d4.csv python tools/profile_trace.py --cuda --reps 1 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:k_timed -s 1 -c 1 --csv --log-file gpurun_out/ncu_d4_exhaust.csv python tools/profile_trace.py --level exhaust --reps 2 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:k_timed -s 1 -c 1 --csv --log-file gpurun_out/ncu_d4_overcommit.csv python tools/profile_trace.py --level overcommit --reps 2 > /dev/null 2>&1
for s in 256 2048 8192; do
  timeout 600 ncu --metrics $M --clock-control none -k regex:k_timed -s 1 -c 1 --csv --log-file gpurun_out/ncu_d3_$s.csv python tools/profile_trace.py --workload d3 --size $s --reps 2 > /dev/null 2>&1
done
grep -c . gpurun_out/sanitize.log; tail -40 gpurun_out/liveness.log
