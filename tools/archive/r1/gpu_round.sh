# Round measurement: tests, smoke, default bench, launch list, one ncu --set full of the top kernel.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1; echo bench_rc=$?; tail -c 4000 gpurun_out/bench_default.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --variant sell:1 > gpurun_out/ncu_bench.log 2>&1; echo ncu_list_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_top ${PROF_ARGS:-python tools/prof_run.py --workload lap8192 --variants sell --reps 1} > gpurun_out/ncu_top.log 2>&1; echo ncu_full_rc=$?
