# multi-line pattern tiles: debug-trap build parity, then timing of (K, line bytes, stages) builds
mkdir -p gpurun_out
PEPP_NVCC_EXTRA="-DPEPP_TILE_CHECKS=1" python build.py --force > /dev/null 2>&1; echo build_checks_rc=$?
timeout 1200 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_fullsize.py -q -p no:cacheprovider -k "ptile or config4" > gpurun_out/mtile_pytest.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/mtile_pytest.log; grep ^FAILED gpurun_out/mtile_pytest.log
timeout 600 python tools/sanitize_run.py > gpurun_out/mtile_sanrun.log 2>&1; echo sanrun_rc=$?; tail -1 gpurun_out/mtile_sanrun.log
for cfg in "" "-DPEPP_MTILE_K=1" "-DPEPP_MTILE_K=6 -DPEPP_PTILE_S=3" "-DPEPP_MTILE_K=8 -DPEPP_PTILE_S=2" "-DPEPP_MTILE_K=2 -DPEPP_MTILE_LINE_KB=16" "-DPEPP_MTILE_K=3 -DPEPP_MTILE_LINE_KB=16 -DPEPP_PTILE_S=2"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:1 8192:f32:1 4096:f64:1 2>&1
done
