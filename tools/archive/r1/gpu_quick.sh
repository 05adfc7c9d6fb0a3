# quick check: SELL parity + default bench (headline + value-compressed leg)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py -q -x > gpurun_out/pytest_quick.log 2>&1; echo pytest_rc=$?; tail -2 gpurun_out/pytest_quick.log
timeout 600 python bench.py --no-sweep --no-cpu > gpurun_out/bench_quick.log 2>&1; echo bench_rc=$?; tail -1 gpurun_out/bench_quick.log
