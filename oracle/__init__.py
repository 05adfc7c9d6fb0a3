"""TEST INFRASTRUCTURE ONLY — the CPU oracle for the SpMV hot path.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package. The
product path (``paper_conf_sc_dastgeerlk12_b200``) never imports it and shares
no code with it.

Every function is a thin ctypes call into ``oracle/oracle.c`` (plain C,
``-O2 -ffp-contract=off``); see that file's header for the paper passages each
one follows. Pins: ``tests/test_oracle_pins.py`` (dense brute force,
permutation, diagonal, Laplacian closed forms, exact-sum bound, power-of-two
scaling, partition brute force) — none of them re-calls this code to make its
expected value. The tolerance and checker helpers (``bound``, ``bound_rows``,
``bound_f32``, ``abs_rowsum``, ``iterate_bound``, ``within``, ``equal``) are
pinned by ``tests/test_oracle_bound_pins.py`` against the hand-worked values
of ``tests/golden/bounds_worked.txt`` and by sensitivity cases (a dropped
term, or an error of 2x the bound, must be rejected).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC",
          "-std=c11", "-Wall", "-Wno-unknown-pragmas"]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", _LIB, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        i64 = ctypes.c_int64
        p = ctypes.c_void_p
        L.oracle_spmv_seq.argtypes = [i64, i64, p, p, p, p, p]
        L.oracle_spmv_rows_parallel.argtypes = [i64, i64, p, p, p, p, p]
        L.oracle_spmv_row.argtypes = [i64, i64, p, p, p, p]
        L.oracle_spmv_row.restype = ctypes.c_double
        L.oracle_abs_rowsum.argtypes = [i64, i64, p, p, p, p, p]
        L.oracle_abs_row.argtypes = [i64, i64, p, p, p, p]
        L.oracle_abs_row.restype = ctypes.c_double
        L.oracle_spmv_iterate.argtypes = [i64, i64, i64, p, p, p, p, p, p, p]
        L.oracle_partition_nnz.argtypes = [i64, i64, p, i64, p]
        L.oracle_spmv_seq_f32.argtypes = [i64, i64, p, p, p, p, p]
        L.oracle_spmv_rows_parallel_f32.argtypes = [i64, i64, p, p, p, p, p]
        L.oracle_abs_rowsum_f32.argtypes = [i64, i64, p, p, p, p, p]
        _lib = L
    return _lib


def _c(a, dt):
    a = np.ascontiguousarray(a, dtype=dt)
    return a


def _args(row_ptr, col, val):
    rp = _c(row_ptr, np.int64)
    c = _c(col, np.int32)
    v = _c(val, np.float64)
    return rp, c, v


def _ptr(a):
    return a.ctypes.data if a.size else None


def spmv(A, x, parallel: bool = False) -> np.ndarray:
    """y = A·x for a CSR (gen.CSR-like: nrows, row_ptr, col, val) — the definition.
    float32 values select the fp32 instance (fp32 x, products and sums)."""
    if np.asarray(A.val).dtype == np.float32:
        return spmv_f32(A, x, parallel)
    rp, c, v = _args(A.row_ptr, A.col, A.val)
    xx = _c(x, np.float64)
    y = np.empty(A.nrows, dtype=np.float64)
    f = lib().oracle_spmv_rows_parallel if parallel else lib().oracle_spmv_seq
    if A.nrows:
        f(A.nrows, int(rp[0]), _ptr(rp), _ptr(c), _ptr(v), _ptr(xx), _ptr(y))
    return y


def spmv_f32(A, x, parallel: bool = False) -> np.ndarray:
    """The fp32 instance of the definition (paper's `float` signature)."""
    rp = _c(A.row_ptr, np.int64)
    c = _c(A.col, np.int32)
    v = _c(A.val, np.float32)
    xx = _c(x, np.float32)
    y = np.empty(A.nrows, dtype=np.float32)
    f = lib().oracle_spmv_rows_parallel_f32 if parallel else lib().oracle_spmv_seq_f32
    if A.nrows:
        f(A.nrows, int(rp[0]), _ptr(rp), _ptr(c), _ptr(v), _ptr(xx), _ptr(y))
    return y


def bound_f32(A, x) -> np.ndarray:
    """Per-row tolerance for the fp32 instance: 2·nnz_row·2^-23·Σ|a||x|
    (the north-star bound with fp32's unit roundoff 2^-24 in place of 2^-53)."""
    rp = _c(A.row_ptr, np.int64)
    c = _c(A.col, np.int32)
    v = _c(A.val, np.float32)
    xx = _c(x, np.float32)
    s = np.empty(A.nrows, dtype=np.float64)
    if A.nrows:
        lib().oracle_abs_rowsum_f32(A.nrows, int(rp[0]), _ptr(rp), _ptr(c), _ptr(v), _ptr(xx), _ptr(s))
    return 2.0 * row_lengths(A).astype(np.float64) * 2.0 ** -23 * s


def spmv_rows(A, x, rows) -> np.ndarray:
    """y_i for sampled rows i only (full-size parity)."""
    rp, c, v = _args(A.row_ptr, A.col, A.val)
    xx = _c(x, np.float64)
    L = lib()
    first = int(rp[0])
    return np.array([L.oracle_spmv_row(int(i), first, _ptr(rp), _ptr(c), _ptr(v), _ptr(xx))
                     for i in rows], dtype=np.float64)


def bound_rows(A, x, rows) -> np.ndarray:
    """The per-row tolerance of `bound` for sampled rows only."""
    rp, c, v = _args(A.row_ptr, A.col, A.val)
    xx = _c(x, np.float64)
    L = lib()
    first = int(rp[0])
    out = np.empty(len(rows))
    for j, i in enumerate(rows):
        n = int(rp[i + 1] - rp[i])
        out[j] = 2.0 * n * 2.0 ** -52 * L.oracle_abs_row(int(i), first, _ptr(rp), _ptr(c), _ptr(v), _ptr(xx))
    return out


def abs_rowsum(A, x) -> np.ndarray:
    """S_i = Σ |a_ij||x_j| (bound ingredient)."""
    rp, c, v = _args(A.row_ptr, A.col, A.val)
    xx = _c(x, np.float64)
    s = np.empty(A.nrows, dtype=np.float64)
    if A.nrows:
        lib().oracle_abs_rowsum(A.nrows, int(rp[0]), _ptr(rp), _ptr(c), _ptr(v), _ptr(xx), _ptr(s))
    return s


def row_lengths(A) -> np.ndarray:
    return np.diff(np.asarray(A.row_ptr, dtype=np.int64))


def bound(A, x) -> np.ndarray:
    """Per-row tolerance of BASELINE.json north_star: 2·nnz_row·2^-52·Σ|a||x|."""
    return 2.0 * row_lengths(A).astype(np.float64) * 2.0 ** -52 * abs_rowsum(A, x)


def iterate(A, x0, K: int, with_bound: bool = False):
    """x_K = A^K x0 (reading A11); optionally z_K = |A|^K |x0| (P7)."""
    rp, c, v = _args(A.row_ptr, A.col, A.val)
    x = _c(x0, np.float64).copy()
    n = A.nrows
    tmp = np.empty(n)
    z = np.empty(n) if with_bound else None
    zt = np.empty(n) if with_bound else None
    lib().oracle_spmv_iterate(K, n, int(rp[0]), _ptr(rp), _ptr(c), _ptr(v), _ptr(x), _ptr(tmp),
                              _ptr(z) if with_bound else None, _ptr(zt) if with_bound else None)
    return (x, z) if with_bound else x


def iterate_bound(A, zK: np.ndarray, K: int) -> np.ndarray:
    """Propagated componentwise bound of P7: 2·K·γ_w·(1+γ_w)^K·(|A|^K|x0|)."""
    w = int(row_lengths(A).max()) if A.nrows else 0
    u = 2.0 ** -53
    g = w * u / (1 - w * u)
    return 2.0 * K * g * (1 + g) ** K * zK


def within(y, ref, tol) -> np.ndarray:
    """Per-element parity verdict (the checker every parity test applies).

    Finite reference entries: ``|y - ref| <= tol`` (tol from ``bound`` /
    ``bound_f32`` / ``iterate_bound``; an empty row has tol 0, so it must be
    exactly 0). Non-finite reference entries (Inf/NaN in x reach the row
    through a stored entry; IEEE-754 propagation is order-independent for a
    row whose only non-finite terms are infinities of one sign or NaN):
    ``y`` must be the same infinity, or NaN where ``ref`` is NaN. A NaN in
    ``y`` against a finite ``ref`` always fails."""
    y = np.asarray(y, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    tol = np.broadcast_to(np.asarray(tol, dtype=np.float64), ref.shape)
    fin = np.isfinite(ref)
    ok = np.zeros(ref.shape, dtype=bool)
    with np.errstate(invalid="ignore"):
        ok[fin] = np.abs(y[fin] - ref[fin]) <= tol[fin]
    nf = ~fin
    ok[nf] = (y[nf] == ref[nf]) | (np.isnan(y[nf]) & np.isnan(ref[nf]))
    return ok


def equal(y, ref) -> np.ndarray:
    """Bit-exact verdict for integer-valued inputs (reading A7: +0 == -0),
    with NaN equal to NaN (non-finite x)."""
    return within(y, ref, 0.0)


def partition_nnz(A, P: int) -> np.ndarray:
    rp = _c(A.row_ptr, np.int64)
    b = np.empty(P + 1, dtype=np.int64)
    lib().oracle_partition_nnz(A.nrows, int(rp[0]), _ptr(rp), P, _ptr(b))
    return b
