# hybrid SELL: where rows leave the layout (PEPP_SELL_CAP), heavy-tailed matrices
mkdir -p gpurun_out
for c in 1024 512 256 128 64; do
  PEPP_SELL_CAP=$c timeout 300 python tools/sigma_sweep.py --workloads skew,zipf4m --sigmas 4096 --reps 6 2>&1 | sed "s/^/cap=$c /"
done
PEPP_SELL_CAP=256 timeout 600 ncu --metrics gpu__time_duration.sum,l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none --csv python tools/prof_run.py --workload skew --variants sell --reps 1 2>&1 | grep -E "sell_kernel|sell_long" | cut -c1-20,100-400
