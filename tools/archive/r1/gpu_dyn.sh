# sorted SELL: static ranges vs dynamically fetched ranges (PEPP_SELL_GROUPS per warp)
mkdir -p gpurun_out
for g in 0 2 4 8 16; do
  for w in zipf4m skew; do
    PEPP_SELL_GROUPS=$g timeout 600 python bench.py --workload $w --steps 5 --no-cpu --no-sweep --variant sell > gpurun_out/dyn_${w}_$g.log 2>&1
    echo "$w groups=$g rc=$? $(tail -1 gpurun_out/dyn_${w}_$g.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["kernel"], d["roofline"]["avg_launch_us"])')"
  done
done
timeout 600 python -m pytest tests/test_gpu_concurrency.py tests/test_gpu_parity.py -q -x 2>&1 | tail -3
