#!/usr/bin/env python3
"""Short driver for ncu: build one bench workload and run each requested
variant a few times through the C-ABI (forced), nothing else on the GPU.

  python tools/prof_run.py --workload lap8192 --variants sell,csr_vector:2 --reps 3
"""
from __future__ import annotations

import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="lap8192")
    ap.add_argument("--variants", default="")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--compress", type=int, default=0,
                    help="opts.compress_values (0 = the bench headline's layout, 1 = pattern-table chunks)")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"], help="value type (f32: the paper's float instance)")
    a = ap.parse_args()
    import numpy as np
    import torch

    import paper_conf_sc_dastgeerlk12_b200 as pepp
    rp = bench.global_rowptr(a.workload)
    R = len(rp) - 1
    A = bench.make_block(a.workload, 0, R)
    x0 = bench.x0_vector(a.workload, A.ncols)
    if a.dtype == "f32":
        import gen
        A = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows, A.name)
        x0 = x0.astype(np.float32)
    plan = pepp.Plan.from_csr(A, compress_values=bool(a.compress))
    xs = torch.from_numpy(x0).cuda()
    y = torch.empty(R, dtype=torch.float32 if a.dtype == "f32" else torch.float64, device="cuda")
    vs = [bench.parse_variant(v) for v in a.variants.split(",") if v] or \
        [pepp.Choice(c.variant, c.param) for c in plan.candidates()]
    for f in vs:
        for _ in range(a.reps):
            plan.exec(xs, y, force=f)
        torch.cuda.synchronize()
        print("ran", f.name, flush=True)
    plan.close()


if __name__ == "__main__":
    main()
