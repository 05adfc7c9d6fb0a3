# value-compressed phase A: L2 prefetch of the next group's x rows (PEPP_PAT_PREFETCH) / group size
mkdir -p gpurun_out
for flags in ""; do
  PEPP_NVCC_EXTRA="$flags" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --steps 3 > gpurun_out/pf.log 2>&1
  echo "[$flags] $(tail -1 gpurun_out/pf.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); v=d["value_compressed"]; print(d["roofline"]["avg_launch_us"], v["avg_launch_us"], v.get("traffic_frac"))')"
done
python build.py --force > /dev/null 2>&1
