#!/usr/bin/env python3
"""Summarise .ncu-rep files (raw page) into one line per kernel launch."""
import csv
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__warps_eligible.avg.per_cycle_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_shared_mem", "launch__grid_size", "lts__t_sector_hit_rate.pct",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "smsp__average_warp_latency_per_inst_issued.ratio",
        "l1tex__lsu_writeback_active_mem_lg.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio"]


def main(paths):
    for p in paths:
        out = subprocess.run(["ncu", "-i", p, "--page", "raw", "--csv", "--print-units", "base"], capture_output=True, text=True).stdout
        rows = list(csv.reader(out.splitlines()))
        if not rows:
            continue
        h = rows[0]
        for r in rows[2:]:
            d = dict(zip(h, r))
            print(f"== {p}: {d.get('Kernel Name','')[:90]}")
            for k in KEYS:
                if k in d:
                    print(f"   {k:70s} {d[k]}")
            stall = {k: d[k] for k in h if k.startswith("smsp__average_warp_latency_issue_stalled") and k.endswith(".ratio")}
            top = sorted(((float(v or 0), k) for k, v in stall.items()), reverse=True)[:6]
            for v, k in top:
                print(f"   stall {k.replace('smsp__average_warp_latency_issue_stalled_','')[:50]:50s} {v:.2f}")


if __name__ == "__main__":
    main(sys.argv[1:])
