# fp32 stencil list: genlist walk concurrent (second stream) vs sequential, alternating builds
mkdir -p gpurun_out
for rep in 1 2; do
for c in 0 1; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_CONCURRENT=$c" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 --dtype f32 > gpurun_out/slist.log 2>&1
  echo "concurrent=$c $(tail -1 gpurun_out/slist.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
done
done
python build.py --force > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_fp32.py tests/test_gpu_concurrency.py -q -x 2>&1 | tail -1
