"""Pins for the oracle's tolerance and checker helpers (CPU only).

The parity tests accept a GPU row when ``oracle.within(y, y_ref, tol)`` holds
with ``tol`` from ``oracle.bound`` / ``bound_rows`` / ``bound_f32`` /
``iterate_bound``. A wrong exponent, a dropped factor or a loosened constant
in any of them would let a wrong kernel pass, so each is pinned here to
something other than itself:

* hand-worked values (``tests/golden/bounds_worked.txt``: signed values and
  signed x, an empty row, unsorted columns; a 1x1 iteration; the 3x3-grid
  Laplacian's ``|A|x0`` worked cell by cell) — exact binary fractions;
* exact rational arithmetic (``fractions.Fraction``) for ``Σ|a||x|`` on
  signed integer-valued inputs;
* sensitivity: a legal other summation order must pass, a row with one
  term dropped or an error of twice the bound must fail;
* IEEE-754 special values through the definition (Inf/NaN in x).

Definitions: BASELINE.json north_star (per-row bound), SURVEY.md §8(c) P6/P7,
the fp32 instance of SURVEY §8(f) f3 (the paper's ``float`` signature,
PAPER.md P@32944).
"""
from __future__ import annotations

import math
import os
import random
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "bounds_worked.txt")


class _M:
    def __init__(self, nrows, ncols, row_ptr, col, val):
        self.nrows, self.ncols = nrows, ncols
        self.row_ptr = np.asarray(row_ptr, dtype=np.int64)
        self.col = np.asarray(col, dtype=np.int32)
        self.val = val if isinstance(val, np.ndarray) else np.asarray(val, dtype=np.float64)
        self.nnz = int(self.row_ptr[-1] - self.row_ptr[0])


def _num(tok: str) -> float:
    if "*2^" in tok:
        m, e = tok.split("*2^")
        return math.ldexp(float(m), int(e))
    return float(tok)


def _golden() -> dict:
    out = {}
    for line in open(GOLDEN):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        k, *v = line.split()
        out[k] = np.array([_num(t) for t in v])
    return out


G = _golden()


def _case_s():
    A = _M(3, 3, [0, 2, 2, 5], [0, 1, 2, 0, 1], [3.0, -4.0, -1.0, 2.0, -0.5])
    x = np.array([-2.0, 0.5, 1.5])
    return A, x


# ------------------------------------------------------ hand-worked values
def test_golden_case_s_definition_and_abs_rowsum():
    A, x = _case_s()
    assert np.array_equal(oracle.spmv(A, x), G["S.y"])
    assert np.array_equal(oracle.abs_rowsum(A, x), G["S.S"])


def test_golden_case_s_bound_fp64():
    A, x = _case_s()
    assert np.array_equal(oracle.bound(A, x), G["S.b64"])
    # the sampled-row form (oracle_abs_row) gives the same values, any row order
    assert np.array_equal(oracle.bound_rows(A, x, [0, 1, 2]), G["S.b64"])
    assert np.array_equal(oracle.bound_rows(A, x, [2, 0]), G["S.b64"][[2, 0]])


def test_golden_case_s_bound_fp32():
    A, x = _case_s()
    A32 = _M(3, 3, A.row_ptr, A.col, A.val.astype(np.float32))
    assert np.array_equal(oracle.bound_f32(A32, x.astype(np.float32)), G["S.b32"])
    # the fp32 definition on the same exact data
    assert np.array_equal(oracle.spmv(A32, x.astype(np.float32)), G["S.y"].astype(np.float32))


def test_golden_case_d_iteration_and_propagated_bound():
    A = _M(1, 1, [0, 1], [0], [2.0])
    x3, z3 = oracle.iterate(A, np.array([-1.0]), 3, with_bound=True)
    assert x3[0] == G["D.x3"][0] and z3[0] == G["D.z3"][0]
    B = oracle.iterate_bound(A, z3, 3)
    assert abs(B[0] / G["D.B"][0] - 1.0) < 1e-14


def test_golden_case_l_laplacian_one_step_bound():
    A = gen.laplacian2d(3)
    x0 = np.arange(1.0, 10.0)
    x1, z1 = oracle.iterate(A, x0, 1, with_bound=True)
    assert np.array_equal(x1, G["L.x1"])
    assert np.array_equal(z1, G["L.z1"])
    B = oracle.iterate_bound(A, z1, 1)
    assert np.all(np.abs(B / (G["L.Bfactor"][0] * G["L.z1"]) - 1.0) < 1e-14)


# ------------------------------------------------ exact rational checks
def _random_signed(rng, m, n, first):
    rp, cols, vals = [first], [], []
    for _ in range(m):
        L = 0 if rng.random() < 0.2 else rng.randint(1, 2 * n)
        for _ in range(L):
            cols.append(rng.randrange(n))                        # duplicates, unsorted
            vals.append(float(rng.choice([-4, -3, -2, -1, 1, 2, 3, 4])))
        rp.append(rp[-1] + L)
    return _M(m, n, rp, cols, vals)


@pytest.mark.parametrize("seed", range(8))
def test_abs_rowsum_signed_exact(seed):
    """S_i = Σ|a||x| with signed a AND signed x (the parity x vectors are
    signed): exact against rationals on integer data; the row form agrees."""
    rng = random.Random(900 + seed)
    m, n = rng.randint(1, 60), rng.randint(1, 60)
    A = _random_signed(rng, m, n, rng.choice([0, 3, 1 << 33]))
    x = np.array([float(rng.randint(-8, 8)) for _ in range(n)])
    assert (x < 0).any()
    first = int(A.row_ptr[0])
    S = oracle.abs_rowsum(A, x)
    for i in range(m):
        ks = range(int(A.row_ptr[i]) - first, int(A.row_ptr[i + 1]) - first)
        exact = sum((abs(Fraction(float(A.val[k]))) * abs(Fraction(float(x[A.col[k]]))) for k in ks), Fraction(0))
        assert Fraction(float(S[i])) == exact
    rows = list(range(m))[::-1]
    assert np.array_equal(oracle.bound_rows(A, x, rows), oracle.bound(A, x)[rows])
    # fp32 ingredient: exact on the same small integers
    A32 = _M(m, n, A.row_ptr, A.col, A.val.astype(np.float32))
    b32 = oracle.bound_f32(A32, x.astype(np.float32))
    nrow = np.diff(A.row_ptr).astype(np.float64)
    assert np.array_equal(b32, np.ldexp(2.0 * nrow * S, -23))


# ------------------------------------------------------------ sensitivity
@pytest.fixture(scope="module")
def real_case():
    A = gen.uniform(3000, 3000, 16, seed=42)
    x = gen.vector(45, gen.REAL, 3000)
    return A, x, oracle.spmv(A, x), oracle.bound(A, x)


def test_checker_accepts_other_legal_orders(real_case):
    """Reversed summation order and the correctly rounded sum (math.fsum) are
    results another correct kernel may return (reading A5): both pass."""
    A, x, yr, b = real_case
    rev = np.empty(A.nrows)
    fs = np.empty(A.nrows)
    for i in range(A.nrows):
        terms = [float(A.val[k]) * float(x[A.col[k]]) for k in range(A.row_ptr[i], A.row_ptr[i + 1])]
        acc = 0.0
        for t in reversed(terms):
            acc = acc + t
        rev[i] = acc
        fs[i] = math.fsum(terms)
    assert oracle.within(rev, yr, b).all()
    assert oracle.within(fs, yr, b).all()
    assert (rev != yr).any()          # the orders really differ somewhere


def test_checker_rejects_dropped_term(real_case):
    A, x, yr, b = real_case
    rp = A.row_ptr
    y = yr.copy()
    dropped = np.empty(A.nrows)
    for i in range(A.nrows):
        k = int(rp[i + 1]) - 1                                # last stored entry
        dropped[i] = float(A.val[k]) * float(x[A.col[k]])
        acc = 0.0
        for kk in range(int(rp[i]), k):
            acc = acc + float(A.val[kk]) * float(x[A.col[kk]])
        y[i] = acc
    big = np.abs(dropped) > 2 * b
    assert big.sum() > 0.99 * A.nrows
    assert not oracle.within(y, yr, b)[big].any()


def test_checker_rejects_twice_the_bound_and_keeps_half(real_case):
    """An error of 2x the north-star bound fails, 1/2 passes. The offsets are
    built from n_i and S_i in the test (64·n·2^-52·S vs 16·n·2^-52·S = 2x and
    1/2 of 2·n·2^-52·S), so a loosened exponent or factor in bound() would
    accept the first."""
    A, x, yr, b = real_case
    n = np.diff(A.row_ptr).astype(np.float64)
    S = oracle.abs_rowsum(A, x)
    hi = np.ldexp(4.0 * n * S, -52)      # 2x the bound
    lo = np.ldexp(1.0 * n * S, -52)      # 1/2 the bound
    assert not oracle.within(yr + hi, yr, b).any()
    assert not oracle.within(yr - hi, yr, b).any()
    assert oracle.within(yr + lo, yr, b).all()


def test_iterate_bound_tightness():
    """P7 at K = 1 is 2·γ_w·(1+γ_w)·z_1: at least twice one ordering's
    worst-case error γ_w·z_1 and no more than 1.001x that (a factor-K or
    exponent mistake falls outside)."""
    A = gen.laplacian2d(16)
    x0 = gen.vector(4, gen.REAL, 256)
    x1, z1 = oracle.iterate(A, x0, 1, with_bound=True)
    B = oracle.iterate_bound(A, z1, 1)
    w, u = 5, 2.0 ** -53
    g = w * u / (1 - w * u)
    r = B / (2 * g * z1)
    assert np.all((r >= 1.0) & (r <= 1.001))
    # and grows linearly in K (2·K·γ·(1+γ)^K)
    B4 = oracle.iterate_bound(A, z1, 4)
    assert np.all(np.abs(B4 / B / 4.0 - 1.0) < 1e-12)


# -------------------------------------------------- non-finite semantics
def test_within_and_equal_special_values():
    ref = np.array([np.inf, -np.inf, np.nan, 1.0, 0.0, 0.0])
    assert oracle.equal(np.array([np.inf, -np.inf, np.nan, 1.0, -0.0, 0.0]), ref).all()
    bad = np.array([-np.inf, np.inf, 1.0, np.nan, 1e-300, np.inf])
    assert not oracle.equal(bad, ref).any()
    # a finite tolerance never admits a non-finite mismatch
    assert not oracle.within(np.array([np.nan, 2.0]), np.array([1.0, np.inf]), 1e300).any()


def test_oracle_ieee_special_values_in_x():
    """Inf/NaN in x propagate through stored entries exactly as the
    definition's products and sums do (IEEE 754): +Inf·2 = +Inf, +Inf·(-1) =
    -Inf, +Inf + (-Inf) = NaN, a stored 0 times Inf = NaN, NaN absorbs; rows
    that do not reference the column stay finite."""
    inf, nan = np.inf, np.nan
    #        row0: 2*x0      row1: -1*x0     row2: x0 - x1(-inf)  row3: 0*x0   row4: x2(nan)+x3  row5: x3
    A = _M(6, 4, [0, 1, 2, 4, 5, 7, 8], [0, 0, 0, 1, 0, 2, 3, 3],
           [2.0, -1.0, 1.0, 1.0, 0.0, 1.0, 1.0, 5.0])
    x = np.array([inf, -inf, nan, 3.0])
    y = oracle.spmv(A, x)
    expect = np.array([inf, -inf, nan, nan, nan, 15.0])
    assert oracle.equal(y, expect).all()
    assert np.isnan(y[2]) and np.isnan(y[3]) and np.isnan(y[4]) and y[5] == 15.0


# ----------------------------------------------- fp32 row-parallel form
def test_rows_parallel_f32_bitwise_equal_seq():
    A = gen.zipf(20000, 20000, seed=46)
    A32 = _M(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32))
    x = gen.vector(48, gen.REAL, 20000).astype(np.float32)
    ys = oracle.spmv(A32, x)
    yp = oracle.spmv(A32, x, parallel=True)
    assert ys.dtype == yp.dtype == np.float32
    assert np.array_equal(ys, yp)
    # and it is the fp32 definition, not fp64 rounded once
    y64 = oracle.spmv(A, x.astype(np.float64))
    assert (ys != y64.astype(np.float32)).any()
