# Round measurement (session 3): tests, smoke, default bench, launch list, ncu --set full of the
# dominant kernels (config 4 headline + value-compressed, config 3 sorted SELL + mid rows), other
# workloads, fp32, config-5 sweep.
mkdir -p gpurun_out
bash tools/gpu_round2.sh
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel|sell_mid" -c 2 -o gpurun_out/prof_sell_zipf python tools/prof_run.py --workload zipf4m --variants sell --reps 1 > gpurun_out/ncu_sell_zipf.log 2>&1; echo ncu_zipf_rc=$?
timeout 2400 python tools/sweep.py --max-rows 1e8 > gpurun_out/sweep.log 2>&1; echo sweep_rc=$?
tail -3 gpurun_out/sweep.log
