# usage: bash tools/r2/prof_stalls.sh <name> <kernel-regex> <prof_run args...>: full capture + stall breakdown
name=$1; kre=$2; shift 2
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$kre -s 1 -c 1 -o gpurun_out/$name -f \
  python tools/prof_run.py "$@" > gpurun_out/$name.ncu.log 2>&1; echo ncu_rc=$?
python tools/ncu_summary.py gpurun_out/$name.ncu-rep > gpurun_out/$name.summary.txt 2>&1
cat gpurun_out/$name.summary.txt
ncu -i gpurun_out/$name.ncu-rep --page raw --csv 2>/dev/null | python -c "
import csv,sys
r=list(csv.reader(sys.stdin)); h=r[0]; v=r[2]
d={a:b for a,b in zip(h,v)}
st=sorted(((k,float(d[k])) for k in d if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued') and d[k].replace('.','').isdigit()), key=lambda t:-t[1])
tot=sum(x for _,x in st) or 1
for k,x in st[:12]: print(f'{x/tot*100:6.1f}%  {k}')
for k in ['dram__throughput.avg.pct_of_peak_sustained_elapsed','smsp__inst_executed.sum','sm__warps_active.avg.pct_of_peak_sustained_active','smsp__issue_active.avg.pct_of_peak_sustained_active']:
    print(k, d.get(k))
"
