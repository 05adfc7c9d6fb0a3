# ncu --set full of SELL on config 3 (zipf4m) after the per-warp slot-balanced ranges
mkdir -p gpurun_out
python build.py > /dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell_zipf2 python tools/prof_run.py --workload zipf4m --variants sell --reps 1 > gpurun_out/ncu_sz2.log 2>&1; echo z=$?
