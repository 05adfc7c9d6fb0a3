# usage: bash tools/r2/prof_one.sh <name> <kernel-regex> <prof_run args...>
# one `ncu --set full` capture of the first matching launch (source-level, lineinfo) + summary
name=$1; kre=$2; shift 2
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$kre -s 1 -c 1 -o gpurun_out/$name -f \
  python tools/prof_run.py "$@" > gpurun_out/$name.ncu.log 2>&1; echo ncu_rc=$?
python tools/ncu_summary.py gpurun_out/$name.ncu-rep > gpurun_out/$name.summary.txt 2>&1
cat gpurun_out/$name.summary.txt
ncu -i gpurun_out/$name.ncu-rep --page details --csv 2>/dev/null | grep -iE "stall|Warp Cycles|Eligible|Issued" | head -30
