# fp32 stencil list at 5 chunks per warp step: GPU suite, smoke, fp32 bench line, ncu of the fp32 list kernel
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log; grep "^FAILED" gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py --dtype f32 --steps 5 --no-cpu --no-sweep > gpurun_out/bench_f32.log 2>&1; echo bench_f32_rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sell_slist|sell_kernel" -c 2 -o gpurun_out/prof_sell_f32 python tools/prof_run.py --workload lap8192 --variants sell --reps 1 --dtype f32 > gpurun_out/ncu_sell_f32.log 2>&1; echo ncu_f32_rc=$?
