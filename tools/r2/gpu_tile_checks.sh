# (1) debug build with bounds traps in sell_tile_kernel: tile tests, full-size config 4 (all layouts), sanitize_run
#     (compute-sanitizer is closed on this pool); (2) side-walk placement experiments (timing only)
mkdir -p gpurun_out
PEPP_NVCC_EXTRA="-DPEPP_TILE_CHECKS=1" python build.py --force > /dev/null 2>&1; echo build_checks_rc=$?
timeout 1500 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_fullsize.py tests/test_gpu_nonfinite.py tests/test_gpu_fp32.py tests/test_gpu_partitioned.py -q -p no:cacheprovider > gpurun_out/tile_checks_pytest.log 2>&1; echo pytest_checks_rc=$?; tail -1 gpurun_out/tile_checks_pytest.log; grep ^FAILED gpurun_out/tile_checks_pytest.log
timeout 900 python tools/sanitize_run.py > gpurun_out/tile_checks_sanrun.log 2>&1; echo sanrun_rc=$?; tail -1 gpurun_out/tile_checks_sanrun.log
for cfg in "" "-DPEPP_EXP_TILE_SIDE=1" "-DPEPP_EXP_TILE_SIDE=2"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== side $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 2>&1
done
