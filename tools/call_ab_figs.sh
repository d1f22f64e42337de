mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/gpu_tests.log
bash tools/ab_gpu.sh
OCCS=8 : 
for lib in paper_conf_ppopp_geladog19_b200/variants/libga_*.so; do n=$(basename $lib .so); r=$(GA_TIMED_OCC=8 GA_LIB=$PWD/$lib timeout 120 python tools/profile_trace.py --workload d4 --reps 8 2>&1 | grep "^rep" | tail -n +3 | awk '{print $3}' | sort -n | awk '{a[NR]=$1} END{print a[int((NR+1)/2)]}'); echo "$n | occ8 d4 | $r" >> gpurun_out/ab.log; done
timeout 900 python tools/fig5.py --out gpurun_out/fig5.json > gpurun_out/fig5.log 2>&1
timeout 900 python tools/fig7.py --sizes 8,16,64,256,512 --out gpurun_out/fig7_small.json > gpurun_out/fig7_small.log 2>&1
