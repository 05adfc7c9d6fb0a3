# pattern-tile kernel: parity, then value-compressed timing for (stages, rows per tile, smem/CTA, block) builds
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ptile.py -x -q -p no:cacheprovider > gpurun_out/ptile_pytest.log 2>&1; echo pytest_rc=$?; tail -2 gpurun_out/ptile_pytest.log
echo "== default"; timeout 600 python tools/r2/vc_time.py 8192:f64 8192:f32 2>&1
for cfg in "$@"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64 8192:f32 2>&1
done
