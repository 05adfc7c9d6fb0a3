#!/usr/bin/env python3
"""Critical-path cost of the halo / interior split (opts.overlap) on ONE GPU.

For the config-4 Laplacian (8192^2) partitioned over P ranks, take a middle
rank's row block (it sends one grid row at each end) and time, back to back
on one stream with the L2-exceeding block:
  whole : the block as one plan (the in-order path's kernel)
  split : head (n rows) + tail (n rows) + interior as three plans, one
          after the other
  concurrent_rK : interior on the caller's stream with K SMs left free,
          head + tail on a high-priority side stream (the overlapped call)
The difference is what the overlap costs on the critical path; what it saves
is the exchange time, which runs beside the interior kernel (not measurable
with one GPU). One JSON line per P.

  python tools/overlap_cost.py [--out gpurun_out/overlap_cost.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--ranks", default="2,4,8")
    ap.add_argument("--reps", type=int, default=40)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "overlap_cost.jsonl"))
    a = ap.parse_args()
    import torch

    import gen
    import paper_conf_sc_dastgeerlk12_b200 as pepp

    n = a.n
    A = gen.laplacian2d(n)
    R = A.nrows
    x = torch.from_numpy(gen.vector(5, gen.REAL, R)).cuda()
    y = torch.empty(R, dtype=torch.float64, device="cuda")
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    fo = open(a.out, "w")

    def timed(calls, reps):
        """median µs of the call sequence, replayed from a CUDA graph so that
        host issue time (Python + ctypes per call) does not count; the
        library issues the overlapped call's launches from C++"""
        for _ in range(30):          # calibration of every plan's selector
            for c in calls:
                c()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for c in calls:
                c()
        g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        return statistics.median(ts)

    for P in [int(p) for p in a.ranks.split(",")]:
        bounds = pepp.partition_rows(A.row_ptr, P)
        rk = P // 2
        r0, r1 = int(bounds[rk]), int(bounds[rk + 1])
        parts = {"whole": [(r0, r1)], "split": [(r0, r0 + n), (r1 - n, r1), (r0 + n, r1 - n)]}
        res = {"P": P, "rank": rk, "block_rows": r1 - r0, "head_rows": n, "tail_rows": n}
        for name, rng in parts.items():
            plans = [(pepp.Plan.from_csr(gen.row_block(A, s, e)), s, e) for s, e in rng]
            calls = [lambda p=p, s=s, e=e: p.exec(x, y[s:e], stream=torch.cuda.current_stream()) for p, s, e in plans]
            res[name + "_us"] = round(timed(calls, a.reps), 2)
            if name == "split":
                res["each_us"] = [round(timed([c], a.reps), 2) for c in calls]
            res[name + "_choices"] = [p.select().name for p, _, _ in plans]
            for p, _, _ in plans:
                p.close()
        # as the overlapped call runs it: interior on the caller's stream (its
        # persistent grid leaving `reserve` SMs), head + tail on a high-priority
        # side stream, fork / join (the exchange itself is not modelled)
        # (round 1 swept the reserve with a PEPP_RESERVE_SMS environment knob;
        # round 2 removed run-time experiment knobs from the library: rebuild
        # with -DPEPP_EXP_RESERVE_SMS=n for a sweep)
        side = torch.cuda.Stream(priority=-1)
        for reserve in (int(os.environ.get("PEPP_EXP_RESERVE_SMS", "0")),):
            inner = pepp.Plan.from_csr(gen.row_block(A, r0 + n, r1 - n))
            edges = [(pepp.Plan.from_csr(gen.row_block(A, s, e)), s, e) for s, e in [(r0, r0 + n), (r1 - n, r1)]]

            def conc():
                main = torch.cuda.current_stream()
                side.wait_stream(main)
                inner.exec(x, y[r0 + n:r1 - n], stream=main)
                for p, s, e in edges:
                    p.exec(x, y[s:e], stream=side)
                main.wait_stream(side)
            res[f"concurrent_r{reserve}_us"] = round(timed([conc], a.reps), 2)
            res[f"interior_r{reserve}_us"] = round(timed([lambda: inner.exec(x, y[r0 + n:r1 - n],
                                                                          stream=torch.cuda.current_stream())], a.reps), 2)
            inner.close()
            for p, _, _ in edges:
                p.close()
        res["split_cost_us"] = round(res["split_us"] - res["whole_us"], 2)
        print(json.dumps(res), flush=True)
        fo.write(json.dumps(res) + "\n")
    fo.close()


if __name__ == "__main__":
    main()
