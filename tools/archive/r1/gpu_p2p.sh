# fused peer-memory halo: two-rank tests on one GPU (CUDA IPC within the device) + bench multirank
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_partitioned.py tests/test_gpu_bench_multirank.py -q -x > gpurun_out/pytest_part.log 2>&1; echo part_rc=$?; tail -15 gpurun_out/pytest_part.log
