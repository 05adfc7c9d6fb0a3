# Final measurement pass (12-consumer stencil tiles): smoke, GPU suite, bench lines, launch list, ncu of the headline kernel
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 2000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log; grep "^FAILED" gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>gpurun_out/bench_default.err; echo bench_rc=$?
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep --no-legs > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_sell.csv python bench.py --steps 2 --warmup 3 --variant sell --no-cpu --no-sweep --no-vc-leg --no-library --no-legs > gpurun_out/ncu_bench_sell.log 2>&1; echo ncu_list_rc=$?
bash tools/r2/prof_one.sh r2_ftile_c0 sell_tile --workload lap8192 --variants sell --reps 2 --compress 0 > /dev/null 2>&1; echo prof0_rc=$?
