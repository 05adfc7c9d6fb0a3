mkdir -p gpurun_out
for cfg in "" "-DPEPP_PAT_MAXLEN=8"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || echo build_failed
  echo "== $cfg"; timeout 900 python tools/r2/nine_point.py 2>&1 | grep '^{'; timeout 600 python tools/r2/vc_time.py 8192:f64:1 8192:f32:1 2>&1 | grep '^{' | cut -c1-80
done
