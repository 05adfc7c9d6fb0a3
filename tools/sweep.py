#!/usr/bin/env python3
"""BASELINE.json config 5: invocation-context sweep.

For banded (half-bandwidth 4) and uniform-random (16/row) square matrices
with 10^4 ... 10^8 rows, build one plan, let the history-based selector
calibrate through ordinary automatic calls, then compare its choice with an
exhaustive per-candidate timing in the same process (mean of several
calls, L2 flushed between calls). Also reports the cold pick: the first call
of a fresh plan whose history file holds the previously swept matrices
(nearest-context prior; the first matrix has none). One JSON line per matrix.

  python tools/sweep.py [--max-rows 1e8] [--out gpurun_out/sweep.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--max-rows", type=float, default=1e8)
    ap.add_argument("--kinds", default="banded,uniform")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.jsonl"))
    ap.add_argument("--reps", type=int, default=7)
    a = ap.parse_args()
    import torch

    import gen
    import paper_conf_sc_dastgeerlk12_b200 as pepp

    sizes = [int(round(10 ** e)) for e in np.arange(4.0, 8.01, 0.5)]
    sizes = [s for s in sizes if s <= a.max_rows]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    fo = open(a.out, "w")
    # one history file shared by the whole sweep: every plan loads what the
    # previous matrices recorded (a cold start borrows the nearest context)
    hist_path = os.path.join(os.path.dirname(a.out), "sweep_history.txt")
    if os.path.exists(hist_path):
        os.unlink(hist_path)
    for idx, R in enumerate(sizes):
        for kind in a.kinds.split(","):
            t0 = time.perf_counter()
            seed = 100 + idx
            A = gen.banded(R, 4, seed=seed) if kind == "banded" else gen.uniform(R, R, 16, seed=seed)
            tgen = time.perf_counter() - t0
            x = torch.from_numpy(gen.vector(seed + 50, gen.REAL, R)).cuda()
            y = torch.empty(R, dtype=torch.float64, device="cuda")
            t0 = time.perf_counter()
            plan = pepp.Plan.from_csr(A, history_path=hist_path)
            tplan = time.perf_counter() - t0
            del A
            reps = a.reps if R > 1_000_000 else 3 * a.reps   # short calls: more samples (cheap)
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]

            def timed(force=None):
                # calls issued back to back (no host sync in between): each L2
                # flush keeps the GPU busy while the host queues the next call,
                # so an event pair brackets the SpMV's device time only, not the
                # host's submission gap (which a per-call sync would add)
                u = None
                for e0, e1 in ev:
                    flush.zero_()
                    e0.record()
                    u = plan.exec(x, y, force=force)
                    e1.record()
                torch.cuda.synchronize()
                ts = [e0.elapsed_time(e1) * 1e3 for e0, e1 in ev]
                # the mean, as the selector's objective (reading A10): short
                # calls time in ~2 µs steps, and a median of quantised samples
                # cannot resolve candidates one step apart, a mean can
                return statistics.fmean(ts), u

            # calibration through ordinary automatic calls (flush between calls);
            # the first call is the cold pick (predicted best from the prior)
            calib_calls = 0
            cold = None
            while True:
                flush.zero_()
                u = plan.exec(x, y)
                if cold is None:
                    cold = u
                calib_calls += 1
                if not u.calibrating or calib_calls > 200:
                    break
            plan.flush_history()
            choice = plan.select()
            # every candidate and the automatic call, interleaved rep by rep
            # (round 2: timing one candidate after another let slow drifts of
            # the clock / DRAM state show up as 20-50 % differences between
            # candidates of ~20 µs calls — the automatic call once timed 17.7
            # µs against 26.7 µs for the same kernel forced)
            forces = [pepp.Choice(c.variant, c.param) for c in plan.candidates()] + [None]
            evs = {i: [] for i in range(len(forces))}
            for _rep in range(reps):
                for i, f in enumerate(forces):
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    flush.zero_()
                    e0.record()
                    plan.exec(x, y, force=f, flags=pepp.EXEC_NO_TIMING)   # no library event records inside the pair
                    e1.record()
                    evs[i].append((e0, e1))
            torch.cuda.synchronize()
            per = {}
            for i, f in enumerate(forces[:-1]):
                per[f.name] = statistics.fmean(e0.elapsed_time(e1) * 1e3 for e0, e1 in evs[i])
            t_auto = statistics.fmean(e0.elapsed_time(e1) * 1e3 for e0, e1 in evs[len(forces) - 1])
            best = min(per, key=per.get)
            info = plan.info()
            plan.close()
            rec = {"rows": R, "kind": kind, "nnz": info["nnz"], "cv": round(info["cv_row"], 3),
                   "chosen": choice.name, "chosen_us": round(per[choice.name], 2), "auto_us": round(t_auto, 2),
                   "best": best, "best_us": round(per[best], 2),
                   "ratio": round(per[choice.name] / per[best], 4), "calibration_calls": calib_calls,
                   "cold_chosen": cold.name, "cold_ratio": round(per[cold.name] / per[best], 4),
                   "prior_key": info["prior_key"],
                   "candidates_us": {k: round(v, 2) for k, v in per.items()},
                   "gen_s": round(tgen, 1), "plan_s": round(tplan, 2),
                   "alg_gbs_best": round(info["algorithmic_bytes"] / per[best] / 1e3, 1)}
            print(json.dumps(rec), flush=True)
            fo.write(json.dumps(rec) + "\n")
            fo.flush()
            del plan
            torch.cuda.empty_cache()
    fo.close()


if __name__ == "__main__":
    main()
