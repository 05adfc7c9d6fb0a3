# stencil list (values streamed): chunks per warp step U per value type, vs the general SELL walk (PEPP_NO_SLIST=1)
mkdir -p gpurun_out
run() {  # $1 = label, env already set
  for dt in f64 f32; do
    timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 --dtype $dt > gpurun_out/slist.log 2>&1
    echo "$1 $dt $(tail -1 gpurun_out/slist.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
  done
}
python build.py --force > /dev/null 2>&1
PEPP_NO_SLIST=1 run general
for u in 2 4 8; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F64=$u -DPEPP_SLIST_U_F32=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  run "slist_U=$u"
done
python build.py --force > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py -q -x 2>&1 | tail -1
