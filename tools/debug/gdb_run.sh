#!/bin/bash
# Run a command under cuda-gdb, interrupt after T seconds, dump where every
# device thread is.  usage: T=60 tools/debug/gdb_run.sh OUT python ...
OUT=$1; shift
mkdir -p gpurun_out
timeout -s INT -k 120 ${T:-60} /usr/local/cuda/bin/cuda-gdb -batch -ex "set pagination off" -ex "set cuda break_on_launch none" -ex run \
    -ex "info cuda kernels" -ex "info cuda threads" -ex "bt" --args "$@" > gpurun_out/$OUT.log 2>&1
grep -v "New Thread\|exited\]\|^rep" gpurun_out/$OUT.log | tail -${LINES_OUT:-80}
