# fp32 stencil list: chunks per step x register cap (min blocks per SM)
mkdir -p gpurun_out
for f in "" "-DPEPP_SLIST_MINB_F32=4" "-DPEPP_SLIST_U_F32=2 -DPEPP_SLIST_MINB_F32=5" "-DPEPP_SLIST_U_F32=6" "-DPEPP_SLIST_U_F32=3 -DPEPP_SLIST_MINB_F32=4"; do
  PEPP_NVCC_EXTRA="$f" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 --dtype f32 > gpurun_out/f32.log 2>&1
  echo "[$f] $(tail -1 gpurun_out/f32.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
done
python build.py --force > /dev/null 2>&1
