#!/usr/bin/env python3
"""Time SELL alone on config-5 banded matrices (b = 4, real values), L2 flushed
between calls, median of 11 back-to-back calls — for build A/B experiments.

  python tools/banded_ab.py --rows 1e7,1e8
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--rows", default="1e7,1e8")
a = ap.parse_args()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for R in [int(float(v)) for v in a.rows.split(",")]:
    A = gen.banded(R, 4, seed=7)
    x = torch.from_numpy(gen.vector(8, gen.REAL, R)).cuda()
    y = torch.empty(R, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL) as plan:
        del A
        f = pepp.Choice(pepp.V_SELL, 0)
        ev = []
        for _ in range(13):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.exec(x, y, force=f)
            e1.record()
            ev.append((e0, e1))
        torch.cuda.synchronize()
        ts = [e0.elapsed_time(e1) * 1e3 for e0, e1 in ev[2:]]
        print(f"banded rows={R} sell median_us={statistics.median(ts):.2f} info={ {k: round(v, 4) if isinstance(v, float) else v for k, v in plan.info().items() if k.startswith('sell_')} }", flush=True)
