# final hybrid rule: full GPU suite + heavy-tailed / config 3 bench lines
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for w in skew zipf4m; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu --no-sweep > gpurun_out/cap5_$w.log 2>&1; echo $w rc=$?
  tail -1 gpurun_out/cap5_$w.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel"], d["roofline"]["avg_launch_us"], d["plan"]["sell_fill"], d.get("library_baseline",{}).get("us_per_spmv"))'
done
