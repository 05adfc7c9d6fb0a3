mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_bench_multirank.py -q -p no:cacheprovider -x --timeout 700 -s > gpurun_out/pytest_bmr.log 2>&1; echo pytest_rc=$?; grep -v "NCCL INFO" gpurun_out/pytest_bmr.log | tail -30
