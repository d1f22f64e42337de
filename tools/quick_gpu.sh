#!/bin/bash
# GPU call: gpu tests + timed-kernel occupancy sweep (d4, d3 16 B / 4 KiB) + one ncu capture.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/gpu_tests.log
: > gpurun_out/occ.log
for occ in ${OCCS:-4 8}; do
  for w in "--workload d4" "--workload d3 --size 16" "--workload d3 --size 256" "--workload d3 --size 4096"; do
    echo "== occ $occ $w" >> gpurun_out/occ.log
    GA_TIMED_OCC=$occ timeout 120 python tools/profile_trace.py $w --reps ${REPS:-4} 2>&1 | tail -2 >> gpurun_out/occ.log
  done
done
if [ -n "$NCU" ]; then
  GA_TIMED_OCC=${NCU_OCC:-4} timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 -f -o gpurun_out/d4_timed \
    python tools/profile_trace.py --reps 2 > gpurun_out/ncu_d4.log 2>&1
fi
