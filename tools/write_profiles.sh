#!/bin/bash
# Turn a tools/round_profile.sh gpurun_out/ into the committed profiles/ files
# (bench line, launch list, ncu summaries with stall reasons and per-function
# attribution, DRAM traffic per launch of the d4 kernel).
set -e
cd "$(dirname "$0")/.."
grep '^{' gpurun_out/bench.log | tail -1 > profiles/r01_bench.json
cp gpurun_out/launches_bench.csv profiles/r01_launches_bench.csv
tmp=$(mktemp -d); (cd $tmp && cuobjdump -xelf all "$OLDPWD/paper_conf_ppopp_geladog19_b200/libga.so" > /dev/null)
for w in d4 d3_16; do
  {
    echo "# ncu --set full, k_timed<GaPolicy,4>, workload $w (tools/profile_trace.py), one B200"
    python tools/ncu_summary.py gpurun_out/${w}_timed.ncu-rep 25
    echo; echo "## stall reasons (warp cycles per issued instruction, by reason)"
    ncu -i gpurun_out/${w}_timed.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h,v=rows[0],rows[2]
for i,n in enumerate(h):
    if 'issue_stalled' in n and n.endswith('per_issue_active.ratio') and float(v[i] or 0)>0.05: print(f'  {n.split(\"stalled_\")[1].split(\"_per\")[0]:24s} {float(v[i]):7.2f}')
for n in ('lts__t_requests_srcunit_tex_op_atom_dot_alu.sum','lts__t_requests_srcunit_tex_op_atom_dot_cas.sum','lts__t_requests_srcunit_tex_op_red.sum','lts__t_requests_srcunit_tex_op_read.sum','lts__t_requests_srcunit_tex_op_write.sum','dram__bytes_read.sum','dram__bytes_write.sum'):
    if n in h: print(f'  {n:48s} {v[h.index(n)]}')
"
    echo; echo "## stall samples and executed instructions by device function (tools/ncu_by_func.py)"
    python tools/ncu_by_func.py gpurun_out/${w}_timed.ncu-rep $tmp/ga_bench.sm_100a.cubin "k_timedINS_8GaPolicyELi4" 2>/dev/null | head -20 || true
  } > profiles/r01_ncu_${w}_k_timed.txt
done
ncu -i gpurun_out/d4_timed.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys,json
rows=list(csv.reader(sys.stdin)); h,u,v=rows[0],rows[1],rows[2]
def b(n):
    x=float(v[h.index(n)]); unit=u[h.index(n)]
    return int(x*{'byte':1,'Kbyte':1e3,'Mbyte':1e6,'Gbyte':1e9}.get(unit,1))
r,w=b('dram__bytes_read.sum'),b('dram__bytes_write.sum')
json.dump({'kernel':'k_timed<GaPolicy,4>','workload':'d4_mixed_pressure (full bench trace, one launch)','dram_bytes_read':r,'dram_bytes_write':w,'traffic_bytes':r+w,'source':'profiles/r01_ncu_d4_k_timed.txt (ncu --set full --clock-control none, dram__bytes_read.sum + dram__bytes_write.sum)'},open('profiles/r01_ncu_traffic.json','w'),indent=1)
"
rm -rf $tmp
