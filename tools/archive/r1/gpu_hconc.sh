# hybrid SELL: mid / long-row kernels concurrent with sell_kernel (removed rows skipped by SELL)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_concurrency.py tests/test_gpu_fp32.py -q -x 2>&1 | tail -2
timeout 300 python tools/sigma_sweep.py --workloads zipf4m,skew,uniform1m --sigmas 0 --reps 8 2>&1 | python -c "import sys,json; [print((d:=json.loads(l))['workload'], d['median_us'], d['min_us'], d['long_rows']) for l in sys.stdin if l.startswith('{')]"
for w in zipf4m skew; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu > gpurun_out/hconc_$w.log 2>&1; echo $w rc=$?
  tail -1 gpurun_out/hconc_$w.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel"], d["roofline"]["avg_launch_us"], d["selector"]["ratio"], d.get("library_baseline",{}).get("us_per_spmv"))'
done
