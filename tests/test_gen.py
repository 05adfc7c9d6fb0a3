"""Generator invariants (CPU). The generator holds no SpMV arithmetic."""
from __future__ import annotations

import numpy as np
import pytest

import gen


def _check_csr(A, sorted_unique=True):
    rp = A.row_ptr
    assert rp.dtype == np.int64 and A.col.dtype == np.int32 and A.val.dtype == np.float64
    assert np.all(np.diff(rp) >= 0)
    assert len(A.col) == A.nnz == len(A.val)
    if A.nnz:
        assert A.col.min() >= 0 and A.col.max() < A.ncols
    if sorted_unique:
        for i in range(0, A.nrows, max(1, A.nrows // 997)):
            c = A.col[rp[i] - rp[0]: rp[i + 1] - rp[0]]
            assert np.all(np.diff(c) > 0)


@pytest.mark.parametrize("n", [1, 2, 3, 7, 64, 100])
def test_laplacian_counts_and_structure(n):
    A = gen.laplacian2d(n)
    assert A.nnz == (5 * n * n - 4 * n if n > 1 else 1) == gen.laplacian2d_nnz(n)
    _check_csr(A)
    assert set(np.unique(A.val).tolist()) <= {4.0, -1.0}
    # symmetric pattern
    for i in range(0, n * n, max(1, n * n // 50)):
        for k in range(A.row_ptr[i], A.row_ptr[i + 1]):
            j = A.col[k]
            assert i in A.col[A.row_ptr[j]:A.row_ptr[j + 1]]


def test_laplacian_8192_nnz_matches_baseline():
    assert gen.laplacian2d_nnz(8192) == 335_511_552
    assert gen.laplacian2d_nnz(64) == 20_224           # config 1


@pytest.mark.parametrize("maker", ["lap", "uni", "zipf", "band"])
def test_slices_equal_rows_of_whole(maker):
    mk = {
        "lap": lambda r0=0, r1=None: gen.laplacian2d(37, r0, r1),
        "uni": lambda r0=0, r1=None: gen.uniform(1500, 900, 16, seed=42, r0=r0, r1=r1),
        "zipf": lambda r0=0, r1=None: gen.zipf(1500, 1500, seed=46, r0=r0, r1=r1),
        "band": lambda r0=0, r1=None: gen.banded(1369, 4, seed=100, r0=r0, r1=r1),
    }[maker]
    W = mk()
    for r0, r1 in [(0, 1), (5, 700), (700, W.nrows), (3, 3)]:
        S = mk(r0, r1)
        B = gen.row_block(W, r0, r1)
        assert np.array_equal(S.row_ptr, B.row_ptr)
        assert np.array_equal(S.col, B.col)
        assert np.array_equal(S.val, B.val)


def test_uniform_exact_k_sorted_unique_reproducible():
    A = gen.uniform(5000, 3000, 16, seed=42)
    assert np.all(np.diff(A.row_ptr) == 16)
    _check_csr(A)
    B = gen.uniform(5000, 3000, 16, seed=42)
    assert np.array_equal(A.col, B.col) and np.array_equal(A.val, B.val)
    C = gen.uniform(5000, 3000, 16, seed=43)
    assert not np.array_equal(A.col, C.col)
    # k > ncols/2 uses the complement path; k == ncols is the full row
    D = gen.uniform(100, 20, 15, seed=1)
    _check_csr(D)
    E = gen.uniform(10, 20, 20, seed=1)
    assert np.all(E.col.reshape(10, 20) == np.arange(20))


def test_uniform_columns_roughly_uniform():
    A = gen.uniform(20000, 1000, 16, seed=3)
    h = np.bincount(A.col, minlength=1000)
    assert h.min() > 0.8 * h.mean() and h.max() < 1.2 * h.mean()


def test_zipf_kmax_reading_a13():
    k = np.arange(1, 436, dtype=np.float64)
    w = k ** -1.5
    mean = (k * w).sum() / w.sum()
    k2 = k[:-1]
    w2 = w[:-1]
    assert mean >= 16 > (k2 * w2).sum() / w2.sum()   # 435 is the smallest K_max with mean >= 16
    A = gen.zipf(200000, 200000, seed=46)
    L = np.diff(A.row_ptr)
    assert L.min() >= 1 and L.max() <= 435
    assert abs(L.mean() - mean) < 0.5
    assert abs((L == 1).mean() - w[0] / w.sum()) < 0.01
    _check_csr(A)


def test_banded_structure():
    A = gen.banded(1000, 4, seed=100)
    L = np.diff(A.row_ptr)
    assert L[4:-4].min() == 9 and L[0] == 5 and L[-1] == 5
    _check_csr(A)


def test_value_modes():
    r = gen.values(1, gen.REAL, 10000)
    assert r.min() >= -1 and r.max() < 1 and np.all(r * 2 ** 52 == np.round(r * 2 ** 52))
    i4 = gen.values(1, gen.INT4, 10000)
    assert set(np.unique(i4).tolist()) == {-4.0, -3.0, -2.0, -1.0, 1.0, 2.0, 3.0, 4.0}
    i8 = gen.values(1, gen.INT8, 10000)
    assert set(np.unique(i8).tolist()) == set(float(v) for v in range(-8, 9))
    # offset = global index: a slice equals the tail of the whole
    assert np.array_equal(gen.values(9, gen.REAL, 50, 100), gen.values(9, gen.REAL, 150)[100:])
