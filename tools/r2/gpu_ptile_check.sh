# pattern tiles: parity (ptile tests, value-compression tests, full-size config 4 in every layout) + timing
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_fp32.py tests/test_gpu_nonfinite.py -q -p no:cacheprovider > gpurun_out/ptile_check.log 2>&1; echo pytest_rc=$?; tail -3 gpurun_out/ptile_check.log; grep ^FAILED gpurun_out/ptile_check.log
timeout 600 python tools/r2/vc_time.py 8192:f64 8192:f32 4096:f64 2>&1
