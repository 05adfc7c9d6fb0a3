# Session re-entry check: GPU tests, smoke, bench with / without value compression.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-sweep > gpurun_out/bench_vc_on.log 2>&1; echo bench_on_rc=$?; tail -1 gpurun_out/bench_vc_on.log
timeout 600 python bench.py --no-sweep --no-cpu --no-value-compression > gpurun_out/bench_vc_off.log 2>&1; echo bench_off_rc=$?; tail -1 gpurun_out/bench_vc_off.log
