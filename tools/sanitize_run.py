#!/usr/bin/env python3
"""Small driver for compute-sanitizer (memcheck / racecheck / synccheck):
every candidate of every variant, plus graphs, containers and the partition
path, on small matrices covering the edge cases (empty rows, ragged tails,
long rows spanning many tiles, unaligned `first`, 16-bit and 32-bit SELL
chunks, sorted SELL windows). Exits non-zero on any parity mismatch.

  compute-sanitizer --tool memcheck python tools/sanitize_run.py
"""
from __future__ import annotations

import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402


def main() -> int:
    import torch

    import paper_conf_sc_dastgeerlk12_b200 as pepp
    rng = np.random.default_rng(0)
    mats = [gen.laplacian2d(37), gen.zipf(5000, 5000, seed=47, val_mode=gen.INT4, kmax=435),
            gen.banded(3001, 4, seed=1, val_mode=gen.INT4), gen.uniform(2000, 70000, 9, seed=3, val_mode=gen.INT4)]
    # a long row (spans many merge tiles and CSR-stream pieces) among short and empty rows
    rows = [[(int(c), float(rng.integers(-4, 5))) for c in rng.integers(0, 3000, 9000)], [], [(5, 2.0)]] + \
           [[(i % 3000, 1.0)] if i % 3 else [] for i in range(400)]
    rp = [0]
    cols, vals = [], []
    for r in rows:
        for c, v in r:
            cols.append(c); vals.append(v)
        rp.append(len(cols))
    mats.append(gen.CSR(len(rows), 3000, np.array(rp, np.int64), np.array(cols, np.int32), np.array(vals), 0, len(rows)))
    mats.append(gen.rebase(mats[1], 7))
    # heavy tail: hybrid SELL with mid-length (warp per row) and segmented long rows
    mats.append(gen.zipf(20_000, 20_000, seed=51, alpha=2.0, kmax=20_000, val_mode=gen.INT4))
    bad = 0
    for A in mats:
        x = gen.vector(3, gen.INT8, A.ncols)
        ref = oracle.spmv(A, x)
        xd = torch.from_numpy(x).cuda()
        y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
        with pepp.Plan.from_csr(A, prune=False) as plan:
            for c in plan.candidates():
                f = pepp.Choice(c.variant, c.param)
                y.fill_(float("nan"))
                plan.exec(xd, y, force=f)
                torch.cuda.synchronize()
                if not np.array_equal(y.cpu().numpy(), ref):
                    print("MISMATCH", A.name, f.name)
                    bad += 1
            g = plan.graph(xd, y, iterations=3, mode=0)
            g.launch()
            torch.cuda.synchronize()
            g.close()
            bad += 0 if np.array_equal(y.cpu().numpy(), ref) else 1
    # containers + dependency tracking across two streams
    A = gen.laplacian2d(64)
    x0 = gen.vector(3, gen.INT8, A.nrows)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    with pepp.Plan.from_csr(A) as plan:
        u, v, w = pepp.Vector(A.nrows, host=x0.copy()), pepp.Vector(A.nrows), pepp.Vector(A.nrows)
        plan.exec_vec(u, v, stream=s1)
        plan.exec_vec(v, w, stream=s2)
        v.scale(2.0, stream=s1)
        bad += 0 if np.array_equal(w.host(pepp.ACCESS_READ), oracle.spmv(A, oracle.spmv(A, x0))) else 1
        for c in (u, v, w):
            c.close()
    # fp32 stencil list (values streamed) + its genlist walk
    A32 = gen.laplacian2d(96)
    A32 = gen.CSR(A32.nrows, A32.ncols, A32.row_ptr, A32.col, A32.val.astype(np.float32), A32.r0, A32.global_nrows, A32.name)
    x32 = gen.vector(3, gen.INT8, A32.ncols).astype(np.float32)
    with pepp.Plan.from_csr(A32, compress_values=False) as plan:
        y32 = torch.full((A32.nrows,), float("nan"), dtype=torch.float32, device="cuda")
        plan.exec(torch.from_numpy(x32).cuda(), y32, force=pepp.Choice(pepp.V_SELL, 0))
        torch.cuda.synchronize()
        bad += 0 if np.array_equal(y32.cpu().numpy(), oracle.spmv(A32, x32)) else 1
    # SELL tiles (bulk-copied ranges, producer / consumer mbarrier ring):
    # pattern tiles and stencil tiles, fp64 and fp32, more tiles than CTAs
    L = gen.laplacian2d(2048)   # long runs: tiles in both layouts
    for dt in (np.float64, np.float32):
        Ld = gen.CSR(L.nrows, L.ncols, L.row_ptr, L.col, L.val.astype(dt), L.r0, L.global_nrows, L.name)
        xl = gen.vector(5, gen.INT8, L.ncols).astype(dt)
        for cz in (True, False):
            with pepp.Plan.from_csr(Ld, compress_values=cz, variant_mask=1 << pepp.V_SELL) as plan:
                yl = torch.full((L.nrows,), float("nan"), dtype=torch.from_numpy(xl).dtype, device="cuda")
                for _ in range(3):
                    plan.exec(torch.from_numpy(xl).cuda(), yl)
                torch.cuda.synchronize()
                ok = plan.info()["sell_ptile_frac"] > 0.5 and np.array_equal(yl.cpu().numpy(), oracle.spmv(Ld, xl) if dt == np.float64 else oracle.spmv_f32(Ld, xl))
                bad += 0 if ok else 1
    # overlapped host batch (copy streams, two device slots)
    with pepp.Plan.from_csr(A) as plan:
        xs = [gen.vector(30 + k, gen.INT8, A.nrows) for k in range(3)]
        ys = [np.full(A.nrows, np.nan) for _ in xs]
        plan.exec_host_batch(xs, ys, iterations=2)
        for xk, yk in zip(xs, ys):
            bad += 0 if np.array_equal(yk, oracle.spmv(A, oracle.spmv(A, xk))) else 1
    # column panels (x > 96 MB, random columns): both panel widths
    W = gen.uniform(20_000, 1 << 24, 8, seed=61, val_mode=gen.INT4)
    xw = gen.vector(62, gen.INT8, W.ncols)
    with pepp.Plan.from_csr(W, variant_mask=1 << pepp.V_PANEL) as plan:
        yw = torch.full((W.nrows,), float("nan"), dtype=torch.float64, device="cuda")
        xwd = torch.from_numpy(xw).cuda()
        for c in plan.candidates():
            plan.exec(xwd, yw, force=pepp.Choice(c.variant, c.param))
            torch.cuda.synchronize()
            bad += 0 if np.array_equal(yw.cpu().numpy(), oracle.spmv(W, xw)) else 1
    print("sanitize_run: mismatches =", bad)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
