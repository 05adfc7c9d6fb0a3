# stencil tiles (values streamed): parity, then timing of both layouts for build variants
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ptile.py tests/test_gpu_fp32.py -x -q -p no:cacheprovider > gpurun_out/stile_pytest.log 2>&1; echo pytest_rc=$?; tail -2 gpurun_out/stile_pytest.log
echo "== default"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f32:0 8192:f64:1 8192:f32:1 2>&1
for cfg in "$@"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f32:0 2>&1
done
