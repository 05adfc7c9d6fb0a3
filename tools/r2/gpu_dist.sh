# Round-2: distribution choice (row a4) + P2P + bench multi-rank, on one GPU with the NCCL stand-in.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_partitioned.py tests/test_gpu_bench_multirank.py -q -p no:cacheprovider -x --timeout 600 > gpurun_out/pytest_dist.log 2>&1; echo pytest_rc=$?; tail -30 gpurun_out/pytest_dist.log
