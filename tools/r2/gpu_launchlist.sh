# ptile tests + the ncu launch list of the bench command (variant forced: see DESIGN §7)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ptile.py -q -p no:cacheprovider > gpurun_out/ptile_pytest.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/ptile_pytest.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_sell.csv python bench.py --steps 2 --warmup 3 --variant sell --no-cpu --no-sweep --no-vc-leg --no-library --no-legs > gpurun_out/ncu_bench_sell.log 2>&1; echo ncu_list_rc=$?
timeout 600 python bench.py --steps 2 --warmup 3 --variant sell --no-cpu --no-sweep --no-vc-leg --no-library --no-legs > gpurun_out/bench_sell_forced.log 2>&1; echo bench_rc=$?; grep '^{' gpurun_out/bench_sell_forced.log | tail -1 | cut -c1-300
