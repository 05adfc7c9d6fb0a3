mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/pytest_gpu.log
for w in lap8192 uniform1m zipf4m; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_$w.log 2>&1; echo bench_${w}_rc=$?
  tail -c 1500 gpurun_out/bench_$w.log | grep -o '"selector".*"clocks"'
done
