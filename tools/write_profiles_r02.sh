#!/bin/bash
# Turn the round-2 profiling call's gpurun_out/ into the committed profiles/ files:
# bench line, launch list, ncu --set full summaries (d4 / d3 16 B) with stall
# reasons and per-function attribution, f4 collective evidence, sanitizer and
# liveness logs, the extra ncu captures (CUDA malloc, d4 exhaust, d3 sizes).
set -e
cd "$(dirname "$0")/.."
LIB=${LIB:-paper_conf_ppopp_geladog19_b200/libga.so}
[ -s gpurun_out/bench_full.json ] && grep '^{' gpurun_out/bench_full.json | tail -1 > profiles/r02_bench.json
[ -s gpurun_out/launches_bench.csv ] && cp gpurun_out/launches_bench.csv profiles/r02_launches_bench.csv
tmp=$(mktemp -d); LIBA=$(readlink -f "$LIB"); (cd $tmp && cuobjdump -xelf all "$LIBA" > /dev/null)
OCC=${OCC:-3}
for w in d4 d3_16; do
  [ -s gpurun_out/${w}_timed.ncu-rep ] || continue
  {
    echo "# ncu --set full, k_timed<GaPolicy,$OCC>, workload $w (tools/profile_trace.py), one B200, round 2"
    python tools/ncu_summary.py gpurun_out/${w}_timed.ncu-rep 25
    echo; echo "## stall reasons (warp cycles per issued instruction, by reason)"
    ncu -i gpurun_out/${w}_timed.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h,v=rows[0],rows[2]
for i,n in enumerate(h):
    if 'issue_stalled' in n and n.endswith('per_issue_active.ratio') and float(v[i] or 0)>0.05: print(f'  {n.split(\"stalled_\")[1].split(\"_per\")[0]:24s} {float(v[i]):7.2f}')
for n in ('lts__t_requests_srcunit_tex_op_atom_dot_alu.sum','lts__t_requests_srcunit_tex_op_atom_dot_cas.sum','lts__t_requests_srcunit_tex_op_red.sum','lts__t_requests_srcunit_tex_op_read.sum','lts__t_requests_srcunit_tex_op_write.sum','dram__bytes_read.sum','dram__bytes_write.sum','launch__registers_per_thread','sm__warps_active.avg.pct_of_peak_sustained_active'):
    if n in h: print(f'  {n:48s} {v[h.index(n)]}')
"
    echo; echo "## stall samples and executed instructions by device function (tools/ncu_by_func.py)"
    python tools/ncu_by_func.py gpurun_out/${w}_timed.ncu-rep $tmp/ga_bench.sm_100a.cubin "k_timedINS_8GaPolicyELi$OCC" 2>/dev/null | head -24 || true
  } > profiles/r02_ncu_${w}_k_timed.txt
done
if [ -s gpurun_out/d4_timed.ncu-rep ]; then
ncu -i gpurun_out/d4_timed.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys,json
rows=list(csv.reader(sys.stdin)); h,u,v=rows[0],rows[1],rows[2]
def b(n):
    x=float(v[h.index(n)]); un=u[h.index(n)]
    return x*{'byte':1,'Kbyte':1e3,'Mbyte':1e6,'Gbyte':1e9}.get(un,1)
json.dump({'kernel':'k_timed<GaPolicy,$OCC>','workload':'d4_mixed_pressure (full bench trace, one launch)',
           'dram_bytes_read':b('dram__bytes_read.sum'),'dram_bytes_write':b('dram__bytes_write.sum'),
           'traffic_bytes':b('dram__bytes_read.sum')+b('dram__bytes_write.sum'),
           'source':'profiles/r02_ncu_d4_k_timed.txt (ncu --set full --clock-control none, dram__bytes_read.sum + dram__bytes_write.sum)'}, open('profiles/r02_ncu_traffic.json','w'), indent=1)
"
fi
ls gpurun_out/coll_ncu_s*_*.csv > /dev/null 2>&1 && python tools/coll_evidence.py profiles/r02_coll_ncu.json
[ -s gpurun_out/sanitize.log ] && cp gpurun_out/sanitize.log profiles/r02_sanitize.log
[ -s gpurun_out/liveness.log ] && cp gpurun_out/liveness.log profiles/r02_liveness.log
for f in ncu_cuda_malloc_d4 ncu_d4_exhaust ncu_d4_overcommit ncu_d3_256 ncu_d3_2048 ncu_d3_8192; do
  [ -s gpurun_out/$f.csv ] && cp gpurun_out/$f.csv profiles/r02_$f.csv
done
ls -la profiles
