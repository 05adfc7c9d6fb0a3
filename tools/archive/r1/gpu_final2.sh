# Round measurement (session 3, final): GPU suite, smoke, sanitizers, default bench, other workloads,
# fp32, launch list, ncu of the headline kernels.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log; grep "^FAILED" gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
bash tools/gpu_sanitize.sh 2>&1 | grep -E "_rc=|SUMMARY|mismatches"
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1; echo bench_rc=$?
for w in uniform1m zipf4m skew lap64; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_$w.log 2>&1; echo bench_${w}_rc=$?
done
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --no-vc-leg --no-library --variant sell:1 > gpurun_out/ncu_bench.log 2>&1; echo ncu_list_rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_slist|sell_kernel" -c 2 -o gpurun_out/prof_sell python tools/prof_run.py --workload lap8192 --variants sell --reps 1 --compress 0 > gpurun_out/ncu_sell.log 2>&1; echo ncu_sell_rc=$?
