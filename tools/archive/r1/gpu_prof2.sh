mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"csr_stream_tma" -c 1 -o gpurun_out/prof_stream_lap_r1 python tools/prof_run.py --workload lap8192 --variants csr_stream --reps 1 > gpurun_out/ncu_a.log 2>&1; echo a=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"csr_stream_tma|csr_vector" -c 2 -o gpurun_out/prof_zipf_r1 python tools/prof_run.py --workload zipf4m --variants csr_stream,csr_vector:8 --reps 1 > gpurun_out/ncu_b.log 2>&1; echo b=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell_lap_r1 python tools/prof_run.py --workload lap8192 --variants sell --reps 1 > gpurun_out/ncu_c.log 2>&1; echo c=$?
