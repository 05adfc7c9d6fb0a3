# fp64 stencil list with the concurrent genlist walk (PEPP_SLIST_F64=1) vs the single general kernel, alternating
mkdir -p gpurun_out
for rep in 1 2 3; do
for c in 0 1; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_F64=$c" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 > gpurun_out/slist.log 2>&1
  echo "slist_f64=$c $(tail -1 gpurun_out/slist.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
done
done
python build.py --force > /dev/null 2>&1
