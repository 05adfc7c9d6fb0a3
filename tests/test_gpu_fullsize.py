"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (default plan options, automatic per-call selection), on sampled rows
the oracle computes one by one:

* config 4 (Laplacian 8192², 335.5 M nnz): 16 iterations from an integer x₀
  — x₁₆ on sampled rows equals the oracle applied to the GPU's own x₁₅ bit
  for bit, and x₁ equals the oracle on x₀; 100 iterations from a real x₀ —
  single steps k = 1, 50, 100 within the per-row bound using the GPU's own
  x_{k-1} as the oracle input.
* configs 2 and 3: every candidate once plus the auto choice, sampled rows
  within the bound; integer-valued inputs bit-exact.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402


def _sample_rows(R, n=20000, seed=0, extra=()):
    rng = np.random.default_rng(seed)
    rows = set(rng.integers(0, R, n).tolist())
    rows.update(range(min(R, 64)))
    rows.update(range(max(0, R - 64), R))
    rows.update(int(r) for r in extra if 0 <= r < R)
    return np.array(sorted(rows), dtype=np.int64)


@pytest.fixture(scope="module")
def lap8192():
    return gen.laplacian2d(8192)


def test_config4_integer_iterations_bitwise_on_sampled_rows(lap8192):
    A = lap8192
    n = 8192
    R = A.nrows
    rows = _sample_rows(R, extra=[n - 1, n, R - n - 1, R - n, R // 2])
    x0 = gen.vector(3, gen.INT8, R)
    with pepp.Plan.from_csr(A) as plan:
        a = torch.from_numpy(x0).cuda()
        b = torch.empty_like(a)
        c = torch.empty_like(a)
        plan.exec(a, b, flags=pepp.Y_NEXT_INPUT)
        torch.cuda.synchronize()
        x1 = b.cpu().numpy()
        assert np.array_equal(x1[rows], oracle.spmv_rows(A, x0, rows))
        src, dst = b, c
        for _ in range(14):
            plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
            src, dst = dst, src
        torch.cuda.synchronize()
        x15 = src.cpu().numpy()
        plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
        torch.cuda.synchronize()
        x16 = dst.cpu().numpy()
    assert np.abs(x16).max() < 2.0 ** 53
    assert np.array_equal(x16[rows], oracle.spmv_rows(A, x15, rows))


def test_config4_real_iterations_single_steps_within_bound(lap8192):
    A = lap8192
    R = A.nrows
    rows = _sample_rows(R, seed=1)
    x0 = gen.vector(4, gen.REAL, R)
    check = {1, 50, 100}
    with pepp.Plan.from_csr(A) as plan:
        bufs = [torch.from_numpy(x0).cuda(), torch.empty(R, dtype=torch.float64, device="cuda"),
                torch.empty(R, dtype=torch.float64, device="cuda")]
        src = bufs[0]
        prev_host = x0
        for k in range(1, 101):
            dst = bufs[1] if src is not bufs[1] else bufs[2]
            used = plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
            if k in check:
                torch.cuda.synchronize()
                xk = dst.cpu().numpy()
                ref = oracle.spmv_rows(A, prev_host, rows)
                bnd = oracle.bound_rows(A, prev_host, rows)
                assert np.all(np.abs(xk[rows] - ref) <= bnd), (k, used.name)
            if k + 1 in check:
                torch.cuda.synchronize()
                prev_host = dst.cpu().numpy()
            src = dst


@pytest.mark.parametrize("config", ["uniform1m", "zipf4m"])
def test_configs_2_3_every_candidate_on_sampled_rows(config):
    if config == "uniform1m":
        A = gen.uniform(1 << 20, 1 << 20, 16, seed=43, val_mode=gen.INT4)
        Ar = gen.with_values(A, 42, gen.REAL)
    else:
        A = gen.zipf(4 << 20, 4 << 20, seed=47, val_mode=gen.INT4)
        Ar = gen.with_values(A, 46, gen.REAL)
    R = A.nrows
    rows = _sample_rows(R, n=10000, seed=2)
    xi = gen.vector(44, gen.INT8, R)
    xr = gen.vector(45, gen.REAL, R)
    for M, x, exact in ((A, xi, True), (Ar, xr, False)):
        ref = oracle.spmv_rows(M, x, rows)
        bnd = oracle.bound_rows(M, x, rows)
        xd = torch.from_numpy(x).cuda()
        y = torch.empty(R, dtype=torch.float64, device="cuda")
        with pepp.Plan.from_csr(M) as plan:
            forces = [pepp.Choice(c.variant, c.param) for c in plan.candidates()] + [None]
            for f in forces:
                y.fill_(float("nan"))
                used = plan.exec(xd, y, force=f)
                torch.cuda.synchronize()
                got = y.cpu().numpy()[rows]
                if exact:
                    assert np.array_equal(got, ref), used.name
                else:
                    assert np.all(np.abs(got - ref) <= bnd), used.name
