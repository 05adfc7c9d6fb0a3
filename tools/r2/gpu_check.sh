# Round-2 check: smoke, the GPU suite (no -x: every failure listed), default bench line.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2>gpurun_out/bench.err; echo bench_rc=$?; tail -c 6000 gpurun_out/bench.log; tail -5 gpurun_out/bench.err
