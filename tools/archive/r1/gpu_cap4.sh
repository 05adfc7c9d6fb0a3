# hybrid SELL: cap x mid-row limit on the heavy-tailed matrices
mkdir -p gpurun_out
for m in 0 512 1024 2048; do
for c in default 128 64; do
  export PEPP_SELL_MIDMAX=$m
  if [ $c = default ]; then unset PEPP_SELL_CAP; else export PEPP_SELL_CAP=$c; fi
  timeout 300 python tools/sigma_sweep.py --workloads skew,zipf4m --sigmas 0 --reps 6 2>&1 | sed "s/^/mid=$m cap=$c /" >> gpurun_out/cap4.log
done
done
cat gpurun_out/cap4.log | python -c "import sys,json
for l in sys.stdin:
    p,_,j=l.partition(\"{\"); d=json.loads(\"{\"+j); print(p, d[\"workload\"], d[\"long_rows\"], d[\"median_us\"])"
