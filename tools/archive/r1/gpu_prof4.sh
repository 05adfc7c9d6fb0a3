# ncu --set full of SELL on configs 2 and 3 (gather-bound matrices)
mkdir -p gpurun_out
python build.py > /dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell_zipf python tools/prof_run.py --workload zipf4m --variants sell --reps 1 > gpurun_out/ncu_sz.log 2>&1; echo z=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell_unif python tools/prof_run.py --workload uniform1m --variants sell --reps 1 > gpurun_out/ncu_su.log 2>&1; echo u=$?
