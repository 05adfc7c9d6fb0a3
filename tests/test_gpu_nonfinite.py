"""Non-finite x (Inf / NaN) through every candidate, against the oracle.

The definition y_i = Σ_k a_ik·x_col(k) (PAPER.md P@32944 + P@31037) sends a
non-finite x_j only into the rows that store an entry in column j, with
IEEE-754 propagation: ±Inf times a nonzero value stays infinite, a stored 0
times Inf is NaN, Inf + (−Inf) is NaN, NaN absorbs. These results do not
depend on the summation order, so every variant must reproduce the oracle
exactly on those rows (NaN-aware equality, ``oracle.equal``), and every
other row must be untouched by them: padding slots, masked lanes, staged
tiles, carries and pattern / stencil chunks must never multiply a
non-finite x they do not own (0·Inf would turn a finite row into NaN).
Integer-valued matrices and finite x entries keep the finite rows bit-exact;
real values are checked within the north-star bound (``oracle.within``).
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402


def _poison(x, seed, frac=0.002, dt=np.float64):
    x = x.astype(dt).copy()
    rng = np.random.default_rng(seed)
    idx = rng.choice(x.size, max(3, int(frac * x.size)), replace=False)
    kinds = np.array([np.inf, -np.inf, np.nan], dtype=dt)
    x[idx] = kinds[np.arange(idx.size) % 3]
    x[0] = np.inf            # column 0: the padding column of SELL / CSR-stream slots
    return x


def _f32(A):
    return gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows)


def _zero_entries(A, seed):
    """Some stored entries set to 0.0: 0·Inf = NaN must appear exactly there."""
    v = A.val.copy()
    rng = np.random.default_rng(seed)
    v[rng.choice(v.size, max(1, v.size // 500), replace=False)] = 0.0
    return gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, v, A.r0, A.global_nrows)


CASES = {
    "lap64": lambda: gen.laplacian2d(64),
    "lap300": lambda: gen.laplacian2d(300),
    "uniform": lambda: gen.uniform(40_000, 40_000, 16, seed=43, val_mode=gen.INT4),
    "zipf": lambda: gen.zipf(60_000, 60_000, seed=47, val_mode=gen.INT4),          # hybrid SELL rows, merge carries
    "banded": lambda: gen.banded(30_001, 4, seed=100, val_mode=gen.INT4),
    "skew": lambda: gen.zipf(200_000, 200_000, seed=50, alpha=2.0, kmax=150_000, val_mode=gen.INT4),   # long rows
}


@pytest.mark.parametrize("case", sorted(CASES))
@pytest.mark.parametrize("compress", [False, True])
def test_nonfinite_x_every_candidate(case, compress):
    A = _zero_entries(CASES[case](), 7)
    x = _poison(gen.vector(44, gen.INT8, A.ncols), 11)
    ref = oracle.spmv(A, x)
    assert np.isnan(ref).any() and np.isinf(ref).any() and np.isfinite(ref).any()
    xd = torch.from_numpy(x).cuda()
    y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A, prune=False, compress_values=compress) as plan:
        for c in plan.candidates():
            y.fill_(-7.0)
            used = plan.exec(xd, y, force=pepp.Choice(c.variant, c.param))
            torch.cuda.synchronize()
            ok = oracle.equal(y.cpu().numpy(), ref)
            bad = np.flatnonzero(~ok)
            assert bad.size == 0, (used.name, bad[:8], y.cpu().numpy()[bad[:4]], ref[bad[:4]])


@pytest.mark.parametrize("case", ["lap300", "zipf", "skew"])
def test_nonfinite_x_real_values(case):
    A = gen.with_values(CASES[case](), 42, gen.REAL)
    x = _poison(gen.vector(45, gen.REAL, A.ncols), 12)
    ref = oracle.spmv(A, x)
    xf = np.where(np.isfinite(x), x, 0.0)
    tol = oracle.bound(A, np.abs(xf))
    xd = torch.from_numpy(x).cuda()
    y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A, prune=False, compress_values=False) as plan:
        for c in plan.candidates() + [None]:
            f = None if c is None else pepp.Choice(c.variant, c.param)
            y.fill_(-7.0)
            used = plan.exec(xd, y, force=f)
            torch.cuda.synchronize()
            assert oracle.within(y.cpu().numpy(), ref, tol).all(), used.name


@pytest.mark.parametrize("case", ["lap300", "zipf", "banded"])
def test_nonfinite_x_fp32(case):
    A = _f32(_zero_entries(CASES[case](), 8))
    x = _poison(gen.vector(46, gen.INT8, A.ncols), 13, dt=np.float32)
    ref = oracle.spmv(A, x)
    xd = torch.from_numpy(x).cuda()
    y = torch.empty(A.nrows, dtype=torch.float32, device="cuda")
    for compress in (False, True):
        with pepp.Plan.from_csr(A, prune=False, compress_values=compress) as plan:
            for c in plan.candidates():
                y.fill_(-7.0)
                used = plan.exec(xd, y, force=pepp.Choice(c.variant, c.param))
                torch.cuda.synchronize()
                assert oracle.equal(y.cpu().numpy(), ref).all(), (used.name, compress)
