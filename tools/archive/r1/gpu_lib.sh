# cuSPARSE cross-check test + bench lines with the library context
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_cusparse.py -q > gpurun_out/pytest_cusparse.log 2>&1; echo cusparse_rc=$?; tail -3 gpurun_out/pytest_cusparse.log
timeout 600 python bench.py --no-cpu --no-sweep > gpurun_out/bench_lib.log 2>&1; echo bench_rc=$?; tail -1 gpurun_out/bench_lib.log
for w in uniform1m zipf4m skew; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu --no-sweep > gpurun_out/bench_lib_$w.log 2>&1; echo bench_${w}_rc=$?
done
