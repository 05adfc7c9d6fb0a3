# walks beside the tile kernels: blocks per SM
mkdir -p gpurun_out
echo "== default"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 2>&1
for cfg in "$@"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 2>&1
done
