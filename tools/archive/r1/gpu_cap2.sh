# hybrid SELL with the share-based cap: parity + heavy-tailed timings + selection
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_concurrency.py tests/test_gpu_fp32.py -q -x 2>&1 | tail -3
timeout 300 python tools/sigma_sweep.py --workloads skew,zipf4m,uniform1m --sigmas 0 --reps 6
for w in skew zipf4m; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu --no-sweep > gpurun_out/cap2_$w.log 2>&1; echo $w rc=$?
  tail -1 gpurun_out/cap2_$w.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel"], d["roofline"]["avg_launch_us"], d["plan"], d.get("library_baseline",{}).get("us_per_spmv"))'
done
