mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_partitioned.py tests/test_gpu_ptile.py -q -p no:cacheprovider -k "distribution_choice_agreed_and_bitwise or ptile or interleave" --timeout 300 > gpurun_out/dist4b.log 2>&1; echo rc=$?; tail -2 gpurun_out/dist4b.log; grep ^FAILED gpurun_out/dist4b.log
