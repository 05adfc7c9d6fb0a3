# fp64 stencil list: chunks per warp step (PEPP_SLIST_U_F64), config 4, two repeats
mkdir -p gpurun_out
for rep in 1 2; do
for u in 6 8 12 16; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F64=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 > gpurun_out/u64.log 2>&1
  echo "U=$u $(tail -1 gpurun_out/u64.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
done
done
python build.py --force > /dev/null 2>&1
