# phase-A unroll experiment: lap8192 SELL with value compression, kPatU = 1, 2, 4
for u in 2 4 6; do
  PEPP_NVCC_EXTRA="-DPEPP_PAT_U=$u" python build.py --force > /dev/null 2>&1
  python bench.py --no-cpu --no-sweep --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.load(sys.stdin); print('U', $u, d['value'], d['roofline']['avg_launch_us'])"
done
python build.py --force > /dev/null 2>&1
