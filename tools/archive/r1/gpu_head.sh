# headline refresh after a SELL kernel change: GPU suite, smoke, default bench, launch list, ncu --set full
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1; echo bench_rc=$?
tail -1 gpurun_out/bench_default.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"], d["e2e"]["value"], d["value_compressed"]["avg_launch_us"], d["clocks"])'
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --no-vc-leg --no-library --variant sell:1 > gpurun_out/ncu_bench.log 2>&1; echo ncu_list_rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell python tools/prof_run.py --workload lap8192 --variants sell --reps 1 --compress 0 > gpurun_out/ncu_sell.log 2>&1; echo ncu_sell_rc=$?
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
