mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?
tail -5 gpurun_out/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_lap_r1.csv python tools/prof_run.py --workload lap8192 --reps 2 > gpurun_out/ncu_list.log 2>&1; echo ncu1_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel|csr_vector_kernel|merge_spmv" -c 9 -o gpurun_out/prof_lap_r1 python tools/prof_run.py --workload lap8192 --variants sell,csr_vector:2,merge_path --reps 3 > gpurun_out/ncu_full.log 2>&1; echo ncu2_rc=$?
tail -3 gpurun_out/ncu_full.log
