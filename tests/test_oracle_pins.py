"""Pins for the CPU oracle (SURVEY.md §8(c) P1–P8), CPU only.

Each expected value here comes from something other than the oracle itself:
exact integer / rational arithmetic in pure Python, a hand-worked fixture,
closed forms of the 5-point Laplacian, or invariants of the mathematics.
A dropped term, a wrong sign or index, a transposed operand, a wrong `first`
offset or an accumulating (y += A·x) oracle each fails at least one test.
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

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


class _M:
    """Minimal CSR holder for hand-built matrices."""

    def __init__(self, nrows, ncols, row_ptr, col, val):
        self.nrows, self.ncols = nrows, ncols
        self.row_ptr = np.asarray(row_ptr, dtype=np.int64)
        self.col = np.asarray(col, dtype=np.int32)
        f32 = isinstance(val, np.ndarray) and val.dtype == np.float32
        self.val = val if f32 else np.asarray(val, dtype=np.float64)


def _random_csr(rng: random.Random, m, n, first, int_vals=True, dup=True, unsorted=True, pempty=0.2):
    rp = [first]
    cols, vals = [], []
    for _ in range(m):
        L = 0 if rng.random() < pempty else rng.randint(1, 2 * n)
        for _ in range(L):
            c = rng.randrange(n)
            cols.append(c)
            vals.append(float(rng.choice([-4, -3, -2, -1, 1, 2, 3, 4])) if int_vals
                        else rng.uniform(-1, 1))
        if not dup:
            pass
        rp.append(rp[-1] + L)
    if not unsorted:
        # sort within rows
        for i in range(m):
            a, b = rp[i] - first, rp[i + 1] - first
            pairs = sorted(zip(cols[a:b], vals[a:b]))
            cols[a:b] = [p[0] for p in pairs]
            vals[a:b] = [p[1] for p in pairs]
    return _M(m, n, rp, cols, vals)


def _dense_exact(A: _M, x):
    """Pure-Python exact dense product via Fractions: D[i][j] accumulates duplicates."""
    first = int(A.row_ptr[0])
    y = []
    for i in range(A.nrows):
        D = {}
        for k in range(int(A.row_ptr[i]) - first, int(A.row_ptr[i + 1]) - first):
            j = int(A.col[k])
            D[j] = D.get(j, Fraction(0)) + Fraction(float(A.val[k]))
        y.append(sum((a * Fraction(float(x[j])) for j, a in D.items()), Fraction(0)))
    return y


# ---------------------------------------------------------------- P1 -----
@pytest.mark.parametrize("seed", range(12))
def test_p1_dense_bruteforce_integer_exact(seed):
    rng = random.Random(seed)
    m, n = rng.randint(1, 64), rng.randint(1, 64)
    first = rng.choice([0, 0, 7, 1 << 33])
    A = _random_csr(rng, m, n, first)
    x = np.array([float(rng.randint(-8, 8)) for _ in range(n)])
    y = oracle.spmv(A, x)
    exact = _dense_exact(A, x)
    assert all(Fraction(float(a)) == b for a, b in zip(y, exact))
    # also through a numpy dense matrix (independent of the CSR loop)
    D = np.zeros((m, n))
    for i in range(m):
        for k in range(int(A.row_ptr[i] - first), int(A.row_ptr[i + 1] - first)):
            D[i, A.col[k]] += A.val[k]
    assert np.array_equal(D @ x, y)


@pytest.mark.parametrize("seed", range(6))
def test_p1_real_within_single_order_bound(seed):
    """Real values: |y - exact| <= γ_n·Σ|a||x| (one summation order, Higham 3.1)."""
    rng = random.Random(100 + seed)
    m, n = rng.randint(1, 40), rng.randint(1, 40)
    A = _random_csr(rng, m, n, 0, int_vals=False)
    x = np.array([rng.uniform(-1, 1) for _ in range(n)])
    y = oracle.spmv(A, x)
    exact = _dense_exact(A, x)
    u = 2.0 ** -53
    for i in range(m):
        L = int(A.row_ptr[i + 1] - A.row_ptr[i])
        S = sum(abs(float(A.val[k])) * abs(float(x[A.col[k]]))
                for k in range(int(A.row_ptr[i]), int(A.row_ptr[i + 1])))
        g = L * u / (1 - L * u) if L else 0.0
        err = abs(Fraction(float(y[i])) - exact[i])
        assert err <= Fraction(g * S * (1 + 1e-12)) + Fraction(0), (i, float(err), g * S)
        if L == 0:
            assert y[i] == 0.0 and math.copysign(1.0, y[i]) == 1.0  # A6: +0.0


def test_golden_hand_worked_laplacian_3x3():
    txt = open(os.path.join(GOLDEN, "laplacian3x3.txt")).read().splitlines()
    lines = [l for l in txt if l and not l.startswith("#")]
    i = lines.index("matrix")
    D = np.array([[float(v) for v in lines[i + 1 + r].split()] for r in range(9)])
    x = np.array([float(v) for v in lines[lines.index("x") + 1].split()])
    y_hand = np.array([float(v) for v in lines[lines.index("y") + 1].split()])
    A = gen.laplacian2d(3)
    # generator structure == hand-written dense matrix
    Dg = np.zeros((9, 9))
    for r in range(9):
        for k in range(A.row_ptr[r], A.row_ptr[r + 1]):
            Dg[r, A.col[k]] += A.val[k]
    assert np.array_equal(Dg, D)
    assert np.array_equal(oracle.spmv(A, x), y_hand)


# ---------------------------------------------------------------- P2/P3 --
@pytest.mark.parametrize("n", [1, 17, 1000])
def test_p2_permutation_exact(n):
    A = gen.permutation_matrix(n, seed=5)
    x = gen.vector(9, gen.REAL, n)
    pi = A.col.astype(np.int64)
    assert sorted(pi.tolist()) == list(range(n))
    assert np.array_equal(oracle.spmv(A, x), x[pi])


@pytest.mark.parametrize("n", [1, 33, 1000])
def test_p3_diagonal_exact(n):
    A = gen.diagonal_matrix(n, seed=6)
    x = gen.vector(10, gen.REAL, n)
    assert np.array_equal(oracle.spmv(A, x), A.val * x)   # one rounding: RN(d·x)


# ---------------------------------------------------------------- P4 -----
@pytest.mark.parametrize("n", [2, 3, 32, 64])
def test_p4_laplacian_closed_forms(n):
    A = gen.laplacian2d(n)
    assert A.nnz == 5 * n * n - 4 * n
    r = np.repeat(np.arange(n), n).astype(np.float64)        # grid-row index
    c = np.tile(np.arange(n), n).astype(np.float64)
    ones = np.ones(n * n)
    y1 = oracle.spmv(A, ones)
    # A·1: number of absent neighbours of each cell
    absent = (r == 0).astype(float) + (r == n - 1) + (c == 0) + (c == n - 1)
    assert np.array_equal(y1, absent)
    assert y1.sum() == 4 * n
    # A·r = -[r=0] + n·[r=n-1] + r·([c=0] + [c=n-1])
    yr = oracle.spmv(A, r)
    expect = -(r == 0).astype(float) + n * (r == n - 1) + r * ((c == 0).astype(float) + (c == n - 1))
    assert np.array_equal(yr, expect)


@pytest.mark.parametrize("n,p,q", [(32, 1, 1), (32, 3, 7), (64, 5, 2)])
def test_p4_laplacian_eigenvector(n, p, q):
    A = gen.laplacian2d(n)
    r = np.repeat(np.arange(n), n)
    c = np.tile(np.arange(n), n)
    v = np.sin(np.pi * p * (r + 1) / (n + 1)) * np.sin(np.pi * q * (c + 1) / (n + 1))
    lam = 4 - 2 * np.cos(np.pi * p / (n + 1)) - 2 * np.cos(np.pi * q / (n + 1))
    Av = oracle.spmv(A, v)
    absA_absv = oracle.abs_rowsum(A, np.abs(v))
    assert np.all(np.abs(Av - lam * v) <= 2.0 ** -45 * (absA_absv + lam * np.abs(v)))


# ---------------------------------------------------------------- P5 -----
def test_p5_iterated_laplacian_integer_exact_k16():
    n = 16
    A = gen.laplacian2d(n)
    x0 = gen.vector(3, gen.INT8, n * n)
    # exact integer iteration in pure Python
    xi = [int(v) for v in x0]
    rows = [[(int(A.col[k]), int(A.val[k])) for k in range(A.row_ptr[i], A.row_ptr[i + 1])]
            for i in range(n * n)]
    for _ in range(16):
        xi = [sum(a * xi[j] for j, a in row) for row in rows]
    assert max(abs(v) for v in xi) < 2 ** 53
    xK = oracle.iterate(A, x0, 16)
    assert [int(v) for v in xK] == xi and np.all(xK == np.array(xi, dtype=np.float64))


def test_p7_iterated_real_within_propagated_bound():
    n, K = 6, 8
    A = gen.laplacian2d(n)
    x0 = gen.vector(4, gen.REAL, n * n)
    xK, zK = oracle.iterate(A, x0, K, with_bound=True)
    rows = [[(int(A.col[k]), Fraction(float(A.val[k]))) for k in range(A.row_ptr[i], A.row_ptr[i + 1])]
            for i in range(n * n)]
    xe = [Fraction(float(v)) for v in x0]
    for _ in range(K):
        xe = [sum((a * xe[j] for j, a in row), Fraction(0)) for row in rows]
    # the oracle's own error against exact must sit inside half the P7 bound (one of two orderings)
    b = oracle.iterate_bound(A, zK, K)
    for i in range(n * n):
        assert abs(Fraction(float(xK[i])) - xe[i]) <= Fraction(float(b[i])) / 2
    # z_K = |A|^K |x0| checked exactly for this nonneg iteration
    ze = [abs(Fraction(float(v))) for v in x0]
    absrows = [[(j, abs(a)) for j, a in row] for row in rows]
    for _ in range(K):
        ze = [sum((a * ze[j] for j, a in row), Fraction(0)) for row in absrows]
    assert all(abs(Fraction(float(zK[i])) - ze[i]) <= ze[i] * Fraction(1, 10 ** 12) for i in range(n * n))


# ---------------------------------------------------------------- P8 -----
@pytest.mark.parametrize("s", [-20, 3, 40])
def test_p8_power_of_two_scaling_bitwise(s):
    A = gen.uniform(500, 700, 16, seed=42)
    x = gen.vector(45, gen.REAL, 700)
    y = oracle.spmv(A, x)
    ys = oracle.spmv(A, np.ldexp(x, s))
    assert np.array_equal(ys, np.ldexp(y, s))


def test_first_offset_and_row_blocks_concatenate():
    """A1 + P@27875: blocks with their own `first` concatenate to the whole y."""
    A = gen.zipf(3000, 2000, seed=46, kmax=100)
    x = gen.vector(48, gen.REAL, 2000)
    y = oracle.spmv(A, x)
    b = [0, 1, 700, 701, 2999, 3000]
    parts = [oracle.spmv(gen.row_block(A, b[i], b[i + 1]), x) for i in range(len(b) - 1)]
    assert np.array_equal(np.concatenate(parts), y)
    # rebasing row_ptr by an arbitrary `first` does not change y
    assert np.array_equal(oracle.spmv(gen.rebase(A, 123456789), x), y)
    # y is overwritten, not accumulated (A4): call twice with the same output
    assert np.array_equal(oracle.spmv(A, x), y)


def test_seq_and_rows_parallel_bitwise():
    A = gen.zipf(20000, 20000, seed=46)
    x = gen.vector(48, gen.REAL, 20000)
    assert np.array_equal(oracle.spmv(A, x), oracle.spmv(A, x, parallel=True))


def test_sampled_rows_match_full():
    A = gen.uniform(1000, 1000, 16, seed=42)
    x = gen.vector(45, gen.REAL, 1000)
    y = oracle.spmv(A, x)
    rows = [0, 5, 999, 500]
    assert np.array_equal(oracle.spmv_rows(A, x, rows), y[rows])


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_partition_rule_properties(P):
    A = gen.zipf(5000, 5000, seed=7, kmax=435)
    b = oracle.partition_nnz(A, P)
    rp = A.row_ptr
    Z = A.nnz
    assert b[0] == 0 and b[-1] == A.nrows and np.all(np.diff(b) >= 0)
    maxlen = int(np.diff(rp).max())
    for p in range(P):
        blk = int(rp[b[p + 1]] - rp[b[p]])
        assert blk <= -(-Z // P) + maxlen
        # minimality: the row before bounds[p] is still short of the target
        if 0 < p and b[p] > 0:
            target = -(-p * Z // P)
            assert rp[b[p] - 1] - rp[0] < target <= rp[b[p]] - rp[0]
    # Laplacian: every block within one row length of nnz/P on both ends
    L = gen.laplacian2d(64)
    bl = oracle.partition_nnz(L, 4)
    sizes = np.diff(L.row_ptr[bl])
    assert sizes.max() - sizes.min() <= 2 * 5   # each boundary within one row (<=5 nnz)


# ------------------------------------------------- fp32 instance (f3) ----
@pytest.mark.parametrize("seed", range(6))
def test_f32_oracle_integer_exact_and_real_single_order_bound(seed):
    """The fp32 oracle (paper's `float` signature): exact on small integers
    (all partial sums < 2^24), and within one fp32 summation order of the
    exact rational result on real inputs; it is NOT the fp64 result."""
    rng = random.Random(200 + seed)
    m, n = rng.randint(1, 50), rng.randint(1, 50)
    A = _random_csr(rng, m, n, rng.choice([0, 5]))
    A32 = _M(m, n, A.row_ptr, A.col, A.val.astype(np.float32))
    x = np.array([float(rng.randint(-8, 8)) for _ in range(n)], dtype=np.float32)
    y = oracle.spmv(A32, x)
    assert y.dtype == np.float32
    exact = _dense_exact(A, x.astype(np.float64))
    assert all(Fraction(float(a)) == b for a, b in zip(y, exact))
    # real values: float products and sums, error vs exact within gamma_n(fp32) * S
    R = _random_csr(rng, m, n, 0, int_vals=False)
    R32 = _M(m, n, R.row_ptr, R.col, R.val.astype(np.float32))
    xr = np.array([rng.uniform(-1, 1) for _ in range(n)], dtype=np.float32)
    yr = oracle.spmv(R32, xr)
    ex = _dense_exact(_M(m, n, R.row_ptr, R.col, R32.val.astype(np.float64)), xr.astype(np.float64))
    u = 2.0 ** -24
    for i in range(m):
        L = int(R.row_ptr[i + 1] - R.row_ptr[i])
        S = sum(abs(float(R32.val[k])) * abs(float(xr[R.col[k]])) for k in range(int(R.row_ptr[i]), int(R.row_ptr[i + 1])))
        g = (L * u / (1 - L * u)) if L else 0.0
        assert abs(Fraction(float(yr[i])) - ex[i]) <= Fraction(g * S * (1 + 1e-9))


def test_f32_oracle_rounds_like_float():
    """A case where float and double sums differ: 1 + 2^-24 + 2^-24 is 1 in
    float (each addition rounds) but 1 + 2^-23 in double."""
    A = _M(1, 3, [0, 3], [0, 1, 2], np.array([1.0, 1.0, 1.0], dtype=np.float32))
    x = np.array([1.0, 2.0 ** -24, 2.0 ** -24], dtype=np.float32)
    assert oracle.spmv(A, x)[0] == np.float32(1.0)
    A64 = _M(1, 3, [0, 3], [0, 1, 2], np.array([1.0, 1.0, 1.0]))
    assert oracle.spmv(A64, x.astype(np.float64))[0] == 1.0 + 2.0 ** -23
