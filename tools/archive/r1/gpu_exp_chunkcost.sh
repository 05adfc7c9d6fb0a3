python build.py > /dev/null
for c in 1 2 3 4 5 6; do
  PEPP_SELL_CHUNK_COST=$c python bench.py --workload zipf4m --variant sell --no-cpu --no-sweep --steps 20 --warmup 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.load(sys.stdin); print('cost', $c, d['roofline']['avg_launch_us'])"
done
