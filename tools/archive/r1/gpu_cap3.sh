# hybrid SELL with the warp-per-row mid kernel: caps on the heavy-tailed matrices + parity
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "hybrid or every_variant or edge" 2>&1 | tail -2
for c in default 512 256 128 64 32; do
  if [ $c = default ]; then unset PEPP_SELL_CAP; else export PEPP_SELL_CAP=$c; fi
  timeout 300 python tools/sigma_sweep.py --workloads skew,zipf4m --sigmas 0 --reps 6 2>&1 | sed "s/^/cap=$c /"
done
