# walker warps per tile kind: pattern-tile walkers 4 / 6 / 8 (values-streamed 4)
mkdir -p gpurun_out
for cfg in "" "-DPEPP_TILE_WALKERS_P=6" "-DPEPP_TILE_WALKERS_P=8" "-DPEPP_TILE_WALKERS_P=8 -DPEPP_TILE_WALKERS_S=2"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"; timeout 600 python tools/r2/vc_time.py 8192:f64:0 8192:f64:1 8192:f32:0 8192:f32:1 4096:f64:1 2>&1
done
