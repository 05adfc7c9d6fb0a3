mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench_pinned.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --variant sell:1 > gpurun_out/ncu_bench_pinned.log 2>&1; echo ncu_list_rc=$?
timeout 2400 python tools/sweep.py --max-rows 1e8 > gpurun_out/sweep.log 2>&1; echo sweep_rc=$?
tail -3 gpurun_out/sweep.log
