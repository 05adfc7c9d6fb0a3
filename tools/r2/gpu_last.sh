# Last measurement pass (final build): smoke, GPU suite, bench lines (fp64 / fp32), launch list (variant pinned)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 2000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log; grep "^FAILED" gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>gpurun_out/bench_default.err; echo bench_rc=$?
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep --no-legs > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_sell.csv python bench.py --steps 2 --warmup 3 --variant sell --no-cpu --no-sweep --no-vc-leg --no-library --no-legs > gpurun_out/ncu_bench_sell.log 2>&1; echo ncu_list_rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/dram_sell_c1.csv python tools/prof_run.py --workload lap8192 --variants sell --reps 3 --compress 1 > /dev/null 2>&1; echo dram1_rc=$?
