mkdir -p gpurun_out
bash tools/r2/ab_libs.sh "python tools/r2/vc_time.py 8192:f64 8192:f32 2>&1 | tail -2"
cp tools/r2/libs/lib_b_int.so paper_conf_sc_dastgeerlk12_b200/libpepp_spmv.so
timeout 900 python -m pytest tests/test_gpu_concurrency.py tests/test_gpu_partitioned.py -q -p no:cacheprovider -k "frozen or context_key or iterated_spmv_bitwise" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -p no:cacheprovider -k "compress or lossless or value" 2>&1 | tail -2
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-sweep --no-vc-leg --no-library --no-legs --variant sell:1 > gpurun_out/ncu_bench.log 2>&1; echo ncu_list_rc=$?
