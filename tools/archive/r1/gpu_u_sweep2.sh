# Stencil list chunks per warp step, finer grid around the defaults: fp64 (<= 8-slot sets) U = 10 / 12 / 14,
# fp32 U = 3 / 4 / 5 / 6; config 4, two repeats each (alternating builds)
mkdir -p gpurun_out
row() { tail -1 gpurun_out/usw.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])'; }
for rep in 1 2; do
for u in 10 12 14; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F64=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 > gpurun_out/usw.log 2>&1
  echo "f64 U=$u $(row)"
done
for u in 3 4 5 6; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F32=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --dtype f32 --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 > gpurun_out/usw.log 2>&1
  echo "f32 U=$u $(row)"
done
done
python build.py --force > /dev/null 2>&1
