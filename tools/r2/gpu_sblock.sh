# stencil-tile consumer warps: 8 vs 12, alternating builds, 3 repeats (config 4 values streamed, fp64 / fp32)
mkdir -p gpurun_out
for rep in 1 2 3; do
for cfg in "" "-DPEPP_STILE_BLOCK=416"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > gpurun_out/bc.log 2>&1 || { echo build_failed; continue; }
  echo "== $rep $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f32:0 2>&1 | grep '^{' | cut -c1-75
done; done
