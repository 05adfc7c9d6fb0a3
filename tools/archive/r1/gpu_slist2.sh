# stencil list at the chosen U per value type vs the general walk, alternating, 3 repeats; then the GPU suite
mkdir -p gpurun_out
for rep in 1 2 3; do
  for e in 1 0; do
    for dt in f64 f32; do
      PEPP_NO_SLIST=$e timeout 600 python bench.py --no-cpu --no-sweep --no-vc-leg --no-library --steps 5 --dtype $dt > gpurun_out/slist.log 2>&1
      echo "no_slist=$e $dt $(tail -1 gpurun_out/slist.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["roofline"]["avg_launch_us"], d["value"], d["clocks"]["sm_mhz"])')"
    done
  done
done
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pytest_gpu.log
