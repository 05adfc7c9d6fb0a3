# SELL: two stencil chunks per warp step, A/B per value type (PEPP_SELL_PAIR_F64 / _F32), alternating builds
mkdir -p gpurun_out
for rep in 1 2; do
for f in "-DPEPP_SELL_PAIR_F64=0 -DPEPP_SELL_PAIR_F32=0" "-DPEPP_SELL_PAIR_F64=1 -DPEPP_SELL_PAIR_F32=1"; do
  PEPP_NVCC_EXTRA="$f" python build.py --force > /dev/null 2>&1 || echo build failed
  for dt in f64 f32; do
    timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --steps 5 --dtype $dt > gpurun_out/pair.log 2>&1
    echo "[$f] $dt $(tail -1 gpurun_out/pair.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
  done
done
done
python build.py --force > /dev/null 2>&1
