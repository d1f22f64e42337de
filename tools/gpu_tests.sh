#!/bin/bash
# GPU test tier on the box: one pytest process per test file, each under its
# own timeout (a hung kernel cannot eat the call), then a short bench.
# usage: tools/gpu_tests.sh [test files...]
mkdir -p gpurun_out
: > gpurun_out/gpu_tests.log
FILES=${@:-$(ls tests/test_gpu_*.py)}
for f in $FILES; do
  echo "== $f" >> gpurun_out/gpu_tests.log
  # per-test timeout: a hung kernel kills this file's process after PER_TEST s
  timeout -k 30 ${PER_FILE_TIMEOUT:-900} python -m pytest "$f" -m gpu -q -p no:cacheprovider \
      -o timeout_func_only=false --timeout ${PER_TEST:-180} --timeout-method thread >> gpurun_out/gpu_tests.log 2>&1
  echo "rc=$? $f" >> gpurun_out/gpu_tests.log
done
grep -E "^== |^rc=|passed|failed|error" gpurun_out/gpu_tests.log
if [ -z "$NO_BENCH" ]; then
  timeout 600 python bench.py --steps 10 --warmup 3 --no-extras > gpurun_out/bench_short.json 2> gpurun_out/bench_short.err
  python -c "import json;d=json.load(open('gpurun_out/bench_short.json'));print('bench', d['ms_per_step'], d['value'], 'warm', d['warm'])"
fi
