"""Time one variant (default: sell, forced) of a bench workload: median µs
per SpMV over calls with a 512 MB L2 flush between them (kernel events on the
launching stream), as bench.py's `configs` legs do. A/B tool for builds.

  python tools/r2/wl_time.py zipf4m uniform1m [--variant sell] [--reps 30]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch

import bench
import paper_conf_sc_dastgeerlk12_b200 as pepp

ap = argparse.ArgumentParser()
ap.add_argument("workloads", nargs="+")
ap.add_argument("--variant", default="sell")
ap.add_argument("--reps", type=int, default=30)
a = ap.parse_args()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for wl in a.workloads:
    rp = bench.global_rowptr(wl)
    A = bench.make_block(wl, 0, len(rp) - 1)
    x = torch.from_numpy(bench.x0_vector(wl, A.ncols)).cuda()
    y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A) as plan:
        f = bench.parse_variant(a.variant)
        for _ in range(3):
            plan.exec(x, y, force=f)
        ts = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            u = plan.exec(x, y, force=f)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        print(json.dumps({"workload": wl, "variant": u.name, "us": round(float(np.median(ts)), 2),
                          "launches": u.launches}), flush=True)
