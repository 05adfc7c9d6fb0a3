# configs 2, 3 and the heavy-tailed matrix: bench lines (cuSPARSE context, no CPU oracle)
mkdir -p gpurun_out
for w in uniform1m zipf4m skew; do
  timeout 600 python bench.py --workload $w --steps 5 --no-cpu --no-sweep > gpurun_out/bench_w3_$w.log 2>&1; echo bench_${w}_rc=$?
done
