# Round-2 measurement pass: GPU suite, smoke, sanitizers, default bench, fp32 bench,
# launch list of the bench command, ncu --set full of the headline kernels.
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 2000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log; grep "^FAILED" gpurun_out/pytest_gpu.log
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo ${tool}_rc=$?; tail -2 gpurun_out/sanitize_$tool.log
done
timeout 900 python bench.py > gpurun_out/bench_default.log 2>gpurun_out/bench_default.err; echo bench_rc=$?
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep --no-legs > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --no-vc-leg --no-library --no-legs > gpurun_out/ncu_bench.log 2>&1; echo ncu_list_rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_slist|sell_kernel" -c 2 -o gpurun_out/r2_prof_sell -f python tools/prof_run.py --workload lap8192 --variants sell --reps 1 --compress 0 > gpurun_out/ncu_sell.log 2>&1; echo ncu_sell_rc=$?
