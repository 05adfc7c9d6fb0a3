# walker warps inside the tile kernel: debug-trap parity, then timing for 2 / 0 / 4 walkers
mkdir -p gpurun_out
PEPP_NVCC_EXTRA="-DPEPP_TILE_CHECKS=1" python build.py --force > /dev/null 2>&1; echo build_checks_rc=$?
timeout 1200 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_fullsize.py tests/test_gpu_nonfinite.py tests/test_gpu_parity.py -q -p no:cacheprovider > gpurun_out/walk_pytest.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/walk_pytest.log; grep ^FAILED gpurun_out/walk_pytest.log
timeout 600 python tools/sanitize_run.py > gpurun_out/walk_sanrun.log 2>&1; echo sanrun_rc=$?; tail -1 gpurun_out/walk_sanrun.log
for cfg in "" "-DPEPP_TILE_WALKERS=0" "-DPEPP_TILE_WALKERS=4"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 2>&1
done
