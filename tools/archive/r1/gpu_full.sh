# Full measurement pass: tests, smoke, default bench, other workloads, launch list, top-kernel ncu, config-5 sweep.
mkdir -p gpurun_out
bash tools/gpu_round.sh
for w in uniform1m zipf4m skew lap64; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_$w.log 2>&1; echo bench_${w}_rc=$?
done
timeout 2400 python tools/sweep.py --max-rows 1e8 > gpurun_out/sweep.log 2>&1; echo sweep_rc=$?
