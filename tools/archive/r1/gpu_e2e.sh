# exec_host_batch parity + e2e legs of the default bench and configs 2/3
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "exec_host" 2>&1 | tail -3
timeout 900 python bench.py --no-cpu --no-sweep > gpurun_out/e2e_lap.log 2>&1; echo rc=$?; tail -1 gpurun_out/e2e_lap.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["e2e"])'
for w in uniform1m zipf4m lap64; do
  timeout 600 python bench.py --workload $w --steps 10 --no-cpu --no-sweep > gpurun_out/e2e_$w.log 2>&1; echo $w rc=$?; tail -1 gpurun_out/e2e_$w.log | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["e2e"])'
done
