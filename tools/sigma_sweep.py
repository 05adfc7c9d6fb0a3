#!/usr/bin/env python3
"""Experiment: SELL-C-σ sorting scope on the random-column workloads.
For each σ the plan is restricted to SELL; reports the padding (fill) and the
median kernel time over L2-flushed launches (CUDA events on the stream).

  python tools/sigma_sweep.py --workloads zipf4m,skew --sigmas 1,4096,65536,1048576
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workloads", default="zipf4m,skew")
    ap.add_argument("--sigmas", default="4096,16384,65536,262144,1048576,4194304")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    import numpy as np
    import torch

    import paper_conf_sc_dastgeerlk12_b200 as pepp
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for w in a.workloads.split(","):
        rp = bench.global_rowptr(w)
        R = len(rp) - 1
        A = bench.make_block(w, 0, R)
        x = torch.from_numpy(bench.x0_vector(w, A.ncols)).cuda()
        y = torch.empty(R, dtype=torch.float64, device="cuda")
        st = torch.cuda.current_stream()
        for sg in [int(s) for s in a.sigmas.split(",")]:
            with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, sell_sigma=sg) as plan:
                info = plan.info()
                f = pepp.Choice(pepp.V_SELL, 0)
                ts = []
                for r in range(a.reps + 2):
                    flush.zero_()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(st)
                    plan.exec(x, y, force=f, stream=st)
                    e1.record(st)
                    e1.synchronize()
                    if r >= 2:
                        ts.append(e0.elapsed_time(e1) * 1e3)
                print(json.dumps({"workload": w, "sigma": sg, "plan_sigma": info["sell_sigma"],
                                  "fill": round(info["sell_fill"], 4), "long_rows": info.get("sell_long_rows"),
                                  "median_us": round(float(np.median(ts)), 2), "min_us": round(min(ts), 2)}),
                      flush=True)


if __name__ == "__main__":
    main()
