# stencil list up to 16 slots: banded b = 4 (9 slots) with / without the list, config 4 fp64 / fp32, parity
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_concurrency.py -q -x 2>&1 | tail -1
for e in 1 0; do
  PEPP_NO_SLIST=$e timeout 600 python tools/banded_ab.py --rows 1e7,1e8 2>&1 | grep banded | sed "s/^/no_slist=$e /" | cut -c1-70
done
for dt in f64 f32; do
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 --dtype $dt > gpurun_out/slist.log 2>&1
  echo "config4 $dt $(tail -1 gpurun_out/slist.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
done
