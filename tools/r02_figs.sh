#!/bin/bash
# Fig. 7 (block 256 and the paper's average over blocks 1..1024) and Fig. 5
# (average over blocks) on the current build.
mkdir -p gpurun_out
timeout 1500 python tools/fig7.py --out gpurun_out/r02_fig7.json > gpurun_out/fig7.log 2>&1
timeout 2400 python tools/fig7.py --all-blocks --reps 1 --run-timeout 240 --sizes 16,256,4096,65536,524288 --out gpurun_out/r02_fig7_allblocks.json > gpurun_out/fig7_all.log 2>&1
timeout 1500 python tools/fig5.py --all-blocks --reps 1 --out gpurun_out/r02_fig5_allblocks.json > gpurun_out/fig5_all.log 2>&1
tail -5 gpurun_out/fig7.log gpurun_out/fig7_all.log gpurun_out/fig5_all.log
