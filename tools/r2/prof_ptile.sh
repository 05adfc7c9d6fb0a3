# launch list + one ncu --set full capture of sell_ptile_kernel on config 4 (value-compressed)
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/ptile_launches.csv python tools/prof_run.py --workload lap8192 --variants sell --reps 3 --compress 1 > gpurun_out/ptile_l.log 2>&1; echo list_rc=$?
grep -v "^==" gpurun_out/ptile_launches.csv | python -c "
import csv,sys
for r in csv.DictReader(sys.stdin):
    print(r['Kernel Name'][:60], r['Metric Name'], r['Metric Value'])" | tail -24
bash tools/r2/prof_one.sh ptile sell_ptile --workload lap8192 --variants sell --reps 2 --compress 1
