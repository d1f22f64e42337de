#!/bin/bash
# One ncu --set full capture of the timed kernel (cold heap) + its summary.
# usage: tools/ncu_top.sh NAME [profile_trace.py args...]
NAME=$1; shift
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_timed -s 1 -c 1 \
   -o gpurun_out/$NAME -f python tools/profile_trace.py --reps 2 "$@" > gpurun_out/$NAME.log 2>&1
python tools/ncu_summary.py gpurun_out/$NAME.ncu-rep 40 > gpurun_out/$NAME.txt 2>&1
head -60 gpurun_out/$NAME.txt
