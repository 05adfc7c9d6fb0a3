# value-compressed phase A: chunks per step (PEPP_PAT_U) x gathers in flight (PEPP_PAT_INFLIGHT)
mkdir -p gpurun_out
for f in "" "-DPEPP_PAT_U=8 -DPEPP_PAT_INFLIGHT=40" "-DPEPP_PAT_U=4 -DPEPP_PAT_INFLIGHT=40" "-DPEPP_PAT_U=8 -DPEPP_PAT_INFLIGHT=20" "-DPEPP_PAT_U=16 -DPEPP_PAT_INFLIGHT=80"; do
  PEPP_NVCC_EXTRA="$f" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-library --steps 3 > gpurun_out/pat.log 2>&1
  echo "[$f] $(tail -1 gpurun_out/pat.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); v=d["value_compressed"]; print(v["avg_launch_us"], v.get("traffic_frac"), d["clocks"]["sm_mhz"])')"
done
python build.py --force > /dev/null 2>&1
