# fp64 stencil list: U for long offset sets (banded b = 4) 8 vs 12; config 4 at the new default; parity
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_concurrency.py -q -x 2>&1 | tail -1
for u in 8 12; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F64_LONG=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python tools/banded_ab.py --rows 1e7,1e8 2>&1 | grep banded | sed "s/^/U_long=$u /" | cut -c1-70
done
python build.py --force > /dev/null 2>&1
timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 2>&1 | tail -1 | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print("config4", d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])'
