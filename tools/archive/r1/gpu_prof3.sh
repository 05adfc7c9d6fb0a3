mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"merge_spmv" -c 1 -o gpurun_out/prof_merge_lap python tools/prof_run.py --workload lap8192 --variants merge_path --reps 1 > gpurun_out/ncu_m.log 2>&1; echo m=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"csr_vector" -c 1 -o gpurun_out/prof_vec_zipf python tools/prof_run.py --workload zipf4m --variants csr_vector:8 --reps 1 > gpurun_out/ncu_v.log 2>&1; echo v=$?
