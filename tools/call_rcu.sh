#!/bin/bash
# GPU call: f3 (SRCU + RCU delegation) parity tests, smoke, and the Fig. 6 sweep.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_rcu.py -x -q > gpurun_out/rcu_tests.log 2>&1; echo rc=$? >> gpurun_out/rcu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo rc=$? >> gpurun_out/smoke.log
timeout 1200 python tools/fig6.py --out gpurun_out/fig6.json > gpurun_out/fig6.log 2>&1; echo rc=$? >> gpurun_out/fig6.log
