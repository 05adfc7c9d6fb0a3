mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_hyb.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_hyb.log
for w in skew zipf4m; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu > gpurun_out/bench_hyb_$w.log 2>&1; echo bench_${w}_rc=$?
done
