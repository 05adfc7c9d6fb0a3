# SELL pairing of 16- / 32-bit column chunks too (PEPP_SELL_PAIR_ALL): configs 2, 4, 5-shaped
mkdir -p gpurun_out
for rep in 1 2; do
for f in "-DPEPP_SELL_PAIR_ALL=0" "-DPEPP_SELL_PAIR_ALL=1"; do
  PEPP_NVCC_EXTRA="$f" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 300 python tools/sigma_sweep.py --workloads uniform1m,lap8192 --sigmas 0 --reps 8 2>&1 | python -c "import sys,json; [print(\"$f\", (d:=json.loads(l))[\"workload\"], d[\"median_us\"], d[\"min_us\"]) for l in sys.stdin if l.startswith(\"{\")]"
done
done
PEPP_NVCC_EXTRA="-DPEPP_SELL_PAIR_ALL=1" python build.py --force > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "every_variant or edge or first_offset or determinism" 2>&1 | tail -2
python build.py --force > /dev/null 2>&1
