# consumer warps per tile CTA: 8 (default) / 12 / 6
mkdir -p gpurun_out
for cfg in "" "-DPEPP_PTILE_BLOCK=416" "-DPEPP_PTILE_BLOCK=224"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > gpurun_out/bc.log 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 2>&1 | grep '^{' | cut -c1-90
done
