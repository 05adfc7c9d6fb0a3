# SELL: L2 bulk prefetch of the chunk 1 or 2 steps ahead (PEPP_SELL_PF), fp64 and fp32 config 4, configs 2 / 3
mkdir -p gpurun_out
for pf in 0 1 2; do
  PEPP_NVCC_EXTRA="-DPEPP_SELL_PF=$pf" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --steps 3 > gpurun_out/spf.log 2>&1
  echo "pf=$pf f64 $(tail -1 gpurun_out/spf.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"])')"
  timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --steps 3 --dtype f32 > gpurun_out/spf.log 2>&1
  echo "pf=$pf f32 $(tail -1 gpurun_out/spf.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"])')"
  timeout 300 python tools/sigma_sweep.py --workloads uniform1m,zipf4m --sigmas 0 --reps 6 2>&1 | sed "s/^/pf=$pf /"
done
python build.py --force > /dev/null 2>&1
timeout 600 python bench.py --workload lap64 --steps 5 --no-cpu > gpurun_out/lap64_sel.log 2>&1; tail -1 gpurun_out/lap64_sel.log | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d[\"selector\"])"
