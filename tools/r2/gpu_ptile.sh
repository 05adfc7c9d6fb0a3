# pattern tiles: parity + value-compressed timing on config 4 (fp64 / fp32) and a smaller Laplacian
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_parity.py -k "ptile or compression" -x -q -p no:cacheprovider > gpurun_out/ptile_pytest.log 2>&1; echo pytest_rc=$?; tail -5 gpurun_out/ptile_pytest.log
timeout 600 python tools/r2/vc_time.py 8192:f64 8192:f32 4096:f64 2>&1 | tee gpurun_out/ptile_vc.log
