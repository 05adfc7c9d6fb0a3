# fp32 refresh: sanitizers (incl. the stencil list), fp32 bench line, ncu of the fp32 stencil-list kernel
mkdir -p gpurun_out
bash tools/gpu_sanitize.sh
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
tail -1 gpurun_out/bench_f32.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["avg_launch_us"], d["e2e"]["value"], d["gpu_launches"])'
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_slist|sell_kernel" -c 2 -o gpurun_out/prof_slist_f32 python tools/prof_run.py --workload lap8192 --variants sell --reps 1 --dtype f32 > gpurun_out/ncu_slist.log 2>&1; echo ncu_rc=$?
