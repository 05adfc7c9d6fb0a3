"""One plan, calls on several streams at once (inter-call parallelism,
SURVEY §8(f) f4, paper §IV-E P@21908–27091): the candidates that keep
per-plan device scratch (merge-path and CSR-stream carries, hybrid-SELL
partial sums and their row counters, halo pack buffers) must not let two
in-flight calls interleave on it. Every candidate is forced, four right-hand
sides alternate over two streams with no synchronisation in between, and
every result is compared with the oracle bit for bit (integer-valued
inputs)."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402


def _concurrent(A, nrhs=4, reps=3):
    xs = [gen.vector(20 + i, gen.INT8, A.ncols) for i in range(nrhs)]
    refs = [oracle.spmv(A, x) for x in xs]
    streams = [torch.cuda.Stream() for _ in range(2)]
    with pepp.Plan.from_csr(A) as plan:
        for c in plan.candidates():
            f = pepp.Choice(c.variant, c.param)
            xd = [torch.from_numpy(x).cuda() for x in xs]
            ys = [torch.full((A.nrows,), float("nan"), dtype=torch.float64, device="cuda") for _ in xs]
            torch.cuda.synchronize()
            for _ in range(reps):
                for i in range(nrhs):
                    plan.exec(xd[i], ys[i], force=f, stream=streams[i % 2])
            torch.cuda.synchronize()
            for i in range(nrhs):
                y = ys[i].cpu().numpy()
                bad = np.flatnonzero(y != refs[i])
                assert bad.size == 0, (f.name, i, bad[:8], y[bad[:4]], refs[i][bad[:4]])


def test_two_streams_heavy_tail():
    """Heavy-tailed rows (P(k) ~ k^-2 up to 2^20): merge-path long runs,
    CSR-stream long rows and hybrid-SELL long rows all use plan scratch."""
    A = gen.zipf(1 << 20, 1 << 20, seed=50, alpha=2.0, kmax=1 << 20, val_mode=gen.INT4)
    _concurrent(A)


def test_two_streams_uniform():
    A = gen.uniform(1 << 21, 1 << 21, 16, seed=43, val_mode=gen.INT4)
    _concurrent(A)


def test_reported_launches_match_profiler():
    """pepp_choice_t.launches (the bench's gpu_launches) equals the library
    kernels CUPTI sees for the call, for every candidate of a heavy-tailed
    plan (hybrid SELL: SELL + mid-row + segmented kernels; merge fix-ups;
    CSR-stream fix-up) and of the Laplacian (one SELL kernel)."""
    from torch.profiler import ProfilerActivity, profile
    for A in (gen.zipf(1 << 18, 1 << 18, seed=50, alpha=2.0, kmax=1 << 18, val_mode=gen.INT4), gen.laplacian2d(256)):
        x = torch.from_numpy(gen.vector(3, gen.INT8, A.ncols)).cuda()
        y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
        with pepp.Plan.from_csr(A, prune=False) as plan:
            for c in plan.candidates():
                f = pepp.Choice(c.variant, c.param)
                plan.exec(x, y, force=f)   # warm
                torch.cuda.synchronize()
                with profile(activities=[ProfilerActivity.CUDA]) as prof:
                    u = plan.exec(x, y, force=f)
                    torch.cuda.synchronize()
                seen = sum(e.count for e in prof.key_averages() if "pepp::" in e.key)
                assert u.launches == seen > 0, (A.name, f.name, u.launches, seen)


def test_graph_of_uncalibrated_plan_captures_frozen_choice():
    """pepp_spmv_graph_create on a plan that has timed nothing yet
    captures the frozen choice (best measured, else the static heuristic —
    SELL on the Laplacian: mean <= 12, CV <= 0.5), not the first calibration
    candidate (vector-CSR TPR 2), which would be replayed untimed."""
    from torch.profiler import ProfilerActivity, profile
    A = gen.laplacian2d(256)
    x = torch.from_numpy(gen.vector(3, gen.INT8, A.ncols)).cuda()
    y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A, prune=False) as plan:
        g = plan.graph(x, y, iterations=2, mode=0)
        torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            g.launch()
            torch.cuda.synchronize()
        names = [e.key for e in prof.key_averages() if "pepp::" in e.key]
        g.close()
    assert names and all("sell" in n for n in names), names


def test_context_key_separates_value_type_and_compression():
    """fp32 and value-compressed plans of the same matrix keep
    their own history records (different kernels, ~1.6x apart)."""
    A = gen.laplacian2d(128)
    A32 = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows)
    keys = set()
    for M in (A, A32):
        for cv in (False, True):
            with pepp.Plan.from_csr(M, compress_values=cv) as plan:
                keys.add(plan.info()["key"])
    assert len(keys) == 4
