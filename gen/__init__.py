"""Seeded synthetic CSR inputs (no SpMV arithmetic lives here).

Feeds both the oracle (``oracle/``) and the CUDA path
(``paper_conf_sc_dastgeerlk12_b200``).  Recipes: SURVEY.md §8(d), readings
A12–A16 of SURVEY.md §8(c); DESIGN.md "Input recipe" restates them.

Every array is produced by ``gen/gen.c`` (counter-based SplitMix64), so a
row block ``[r0, r1)`` of any matrix can be generated on its own (one rank's
slice) and equals the same rows of the whole matrix.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "libpepp_gen.so")

# value / vector modes (see gen.c draw_value)
REAL, INT4, INT8, ONES, REAL_NZ = 0, 1, 2, 3, 4


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11",
                               "-Wall", "-Wno-unknown-pragmas", _SRC, "-o", _LIB, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        i64, u64, i32p, i64p, f64p = (ctypes.c_int64, ctypes.c_uint64,
                                      ctypes.POINTER(ctypes.c_int32),
                                      ctypes.POINTER(ctypes.c_int64),
                                      ctypes.POINTER(ctypes.c_double))
        L.gen_u64.restype = u64
        L.gen_u64.argtypes = [u64, u64, u64]
        L.gen_values.argtypes = [u64, ctypes.c_int, i64, i64, f64p]
        L.gen_laplacian2d_nnz.restype = i64
        L.gen_laplacian2d_nnz.argtypes = [i64]
        L.gen_laplacian2d_rowptr.argtypes = [i64, i64, i64, i64p]
        L.gen_laplacian2d_fill.argtypes = [i64, i64, i64, i32p, f64p]
        L.gen_row_lengths.argtypes = [ctypes.c_int, u64, i64, i64, ctypes.c_double, i64, i64, i64, i32p]
        L.gen_lengths_to_rowptr.argtypes = [i64, i32p, i64, i64p]
        L.gen_banded_fill.argtypes = [i64, i64, i64, i64, i64p, i32p]
        L.gen_random_cols_fill.argtypes = [u64, i64, i64, i64, i64p, i32p]
        L.gen_permutation.argtypes = [u64, i64, i32p]
        _lib = L
    return _lib


def _p(a: np.ndarray, t):
    return a.ctypes.data_as(ctypes.POINTER(t))


@dataclass
class CSR:
    """A CSR row block: rows [r0, r1) of an nrows x ncols matrix.

    ``row_ptr`` holds GLOBAL offsets (``row_ptr[0] == first``), i.e. the
    paper's ``first`` convention; ``col``/``val`` hold the
    block's entries only.
    """
    nrows: int          # rows in this block
    ncols: int
    row_ptr: np.ndarray  # int64 [nrows+1], global offsets
    col: np.ndarray      # int32 [nnz]
    val: np.ndarray      # float64 [nnz]
    r0: int = 0
    global_nrows: int = -1
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1] - self.row_ptr[0])

    @property
    def first(self) -> int:
        return int(self.row_ptr[0])


def values(seed: int, mode: int, n: int, offset: int = 0) -> np.ndarray:
    out = np.empty(n, dtype=np.float64)
    if n:
        lib().gen_values(seed, mode, offset, n, _p(out, ctypes.c_double))
    return out


def vector(seed: int, mode: int, n: int) -> np.ndarray:
    """Dense x vector (modes as for values)."""
    return values(seed, mode, n, 0)


def laplacian2d_nnz(n: int) -> int:
    return int(lib().gen_laplacian2d_nnz(n))


def laplacian2d(n: int, r0: int = 0, r1: int | None = None) -> CSR:
    """5-point Laplacian on an n x n grid, rows [r0, r1) (A12)."""
    R = n * n
    r1 = R if r1 is None else r1
    rp = np.empty(r1 - r0 + 1, dtype=np.int64)
    lib().gen_laplacian2d_rowptr(n, r0, r1, _p(rp, ctypes.c_int64))
    z = int(rp[-1] - rp[0])
    col = np.empty(z, dtype=np.int32)
    val = np.empty(z, dtype=np.float64)
    if z:
        lib().gen_laplacian2d_fill(n, r0, r1, _p(col, ctypes.c_int32), _p(val, ctypes.c_double))
    return CSR(r1 - r0, R, rp, col, val, r0, R, f"laplacian2d_{n}")


def _lengths(kind: int, seed: int, nrows: int, ncols: int, alpha: float, k: int, r0: int, r1: int) -> np.ndarray:
    ln = np.empty(r1 - r0, dtype=np.int32)
    if r1 > r0:
        lib().gen_row_lengths(kind, seed, nrows, ncols, alpha, k, r0, r1, _p(ln, ctypes.c_int32))
    return ln


def _rowptr_global(kind, seed, nrows, ncols, alpha, k, r0, r1) -> np.ndarray:
    """Global row_ptr slice for rows [r0, r1]: needs the prefix over [0, r0)."""
    ln_all = _lengths(kind, seed, nrows, ncols, alpha, k, 0, r1)
    first = int(ln_all[:r0].sum(dtype=np.int64))
    rp = np.empty(r1 - r0 + 1, dtype=np.int64)
    lib().gen_lengths_to_rowptr(r1 - r0, _p(np.ascontiguousarray(ln_all[r0:]), ctypes.c_int32),
                                first, _p(rp, ctypes.c_int64))
    return rp


def random_rows(kind: int, seed: int, nrows: int, ncols: int, *, k: int = 16, alpha: float = 1.5,
                kmax: int = 435, val_seed: int | None = None, val_mode: int = REAL,
                r0: int = 0, r1: int | None = None, name: str = "") -> CSR:
    """Random-column matrices: kind 'uniform' (k per row) or 'zipf' (A13)."""
    r1 = nrows if r1 is None else r1
    if kind == "uniform":
        rp = _rowptr_global(0, seed, nrows, ncols, 0.0, k, r0, r1)
    elif kind == "zipf":
        rp = _rowptr_global(1, seed, nrows, ncols, alpha, kmax, r0, r1)
    else:
        raise ValueError(kind)
    z = int(rp[-1] - rp[0])
    col = np.empty(z, dtype=np.int32)
    if z:
        lib().gen_random_cols_fill(seed, ncols, r0, r1, _p(rp, ctypes.c_int64), _p(col, ctypes.c_int32))
    vs = seed + 1 if val_seed is None else val_seed
    val = values(vs, val_mode, z, int(rp[0]))
    return CSR(r1 - r0, ncols, rp, col, val, r0, nrows, name or f"{kind}_{nrows}")


def uniform(nrows: int, ncols: int, k: int, seed: int, **kw) -> CSR:
    return random_rows("uniform", seed, nrows, ncols, k=k, **kw)


def zipf(nrows: int, ncols: int, seed: int, alpha: float = 1.5, kmax: int = 435, **kw) -> CSR:
    return random_rows("zipf", seed, nrows, ncols, alpha=alpha, kmax=kmax, **kw)


def banded(nrows: int, b: int, seed: int, val_mode: int = REAL, r0: int = 0, r1: int | None = None) -> CSR:
    """Square banded matrix, half-bandwidth b (A15)."""
    r1 = nrows if r1 is None else r1
    rp = _rowptr_global(2, seed, nrows, nrows, 0.0, b, r0, r1)
    z = int(rp[-1] - rp[0])
    col = np.empty(z, dtype=np.int32)
    if z:
        lib().gen_banded_fill(nrows, b, r0, r1, _p(rp, ctypes.c_int64), _p(col, ctypes.c_int32))
    val = values(seed, val_mode, z, int(rp[0]))
    return CSR(r1 - r0, nrows, rp, col, val, r0, nrows, f"banded{b}_{nrows}")


def permutation(n: int, seed: int) -> np.ndarray:
    p = np.empty(n, dtype=np.int32)
    if n:
        lib().gen_permutation(seed, n, _p(p, ctypes.c_int32))
    return p


def permutation_matrix(n: int, seed: int) -> CSR:
    """Row i has a single 1.0 at column pi(i): (A x)_i = x[pi(i)] (pin P2)."""
    pi = permutation(n, seed)
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), pi.astype(np.int32),
               np.ones(n), 0, n, f"perm_{n}")


def diagonal_matrix(n: int, seed: int, mode: int = REAL) -> CSR:
    """Row i has d_i at column i (pin P3)."""
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32),
               values(seed, mode, n), 0, n, f"diag_{n}")


def with_values(A: CSR, seed: int, mode: int) -> CSR:
    """Same structure, values redrawn by global nnz index."""
    return CSR(A.nrows, A.ncols, A.row_ptr, A.col, values(seed, mode, A.nnz, A.first),
               A.r0, A.global_nrows, A.name)


def row_block(A: CSR, r0: int, r1: int) -> CSR:
    """Rows [r0, r1) of a whole-matrix CSR, keeping global offsets (paper's `first`)."""
    rp = A.row_ptr[r0:r1 + 1].copy()
    a, b = int(rp[0] - A.row_ptr[0]), int(rp[-1] - A.row_ptr[0])
    return CSR(r1 - r0, A.ncols, rp, A.col[a:b], A.val[a:b], A.r0 + r0,
               A.global_nrows if A.global_nrows >= 0 else A.nrows, A.name)


def rebase(A: CSR, first: int) -> CSR:
    """Same matrix with row_ptr shifted so row_ptr[0] == first (A1)."""
    return CSR(A.nrows, A.ncols, A.row_ptr - A.row_ptr[0] + first, A.col, A.val,
               A.r0, A.global_nrows, A.name)
