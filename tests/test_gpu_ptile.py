"""GPU parity of the SELL tile kernel (sell_tile_kernel): σ = 1 plans compute
runs of stencil chunks from x ranges (and, when the values stream, the
chunks' value block) bulk-copied into shared memory — pattern tiles for
value-compressed plans, stencil tiles over the stencil list otherwise. Per
row the same FMAs in the same slot order as the register paths, so y must
be bit-identical between the layouts and the register paths (and equal to
the oracle on integer inputs, within the north-star bound on real ones).
Covers: 2-D / 3-D stencils (1-5 offset clusters), fp64 and fp32, x / y
views that are not 16-byte aligned (the register path runs instead), tiles
whose ranges would leave x (kept in the phase-A list), and the fraction of
chunks the tiles hold."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402
from test_gpu_parity import _check, _stencil_grid  # noqa: E402


def _y(A, x, compress, dt=torch.float64, shift=0):
    """y through a SELL-only plan; `shift` > 0 runs the call on views that
    start `shift` elements into their buffers (not 16-byte aligned)."""
    with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, prune=False, compress_values=compress) as plan:
        xb = torch.zeros(A.ncols + shift, dtype=dt, device="cuda")
        xb[shift:] = torch.from_numpy(np.ascontiguousarray(x)).to(dt).cuda()
        yb = torch.full((A.nrows + shift,), float("nan"), dtype=dt, device="cuda")
        xv, yv = xb[shift:], yb[shift:]
        for _ in range(3):   # calibration calls, then the measured one
            plan.exec(xv, yv)
        torch.cuda.synchronize()
        return yv.cpu().numpy(), plan.info()


def _bits(a):
    return a.view(np.int64 if a.dtype == np.float64 else np.int32)


@pytest.mark.parametrize("n", [1024, 2048])
def test_ptile_laplacian_bit_identical(n):
    """2048²: both layouts tiled. 1024² (runs of 30 chunks = 960 rows): the
    values-streamed layout is tiled, the value-compressed one keeps the
    register path (pattern tiles need >= 1536 rows per tile on average to pay)."""
    A = gen.laplacian2d(n)
    for x in (gen.vector(3, gen.INT8, A.ncols), gen.vector(4, gen.REAL, A.ncols)):
        y1, i1 = _y(A, x, True)
        y0, i0 = _y(A, x, False)
        assert i0["sell_ptile_frac"] > 0.9
        if n == 2048:
            assert i1["sell_ptile_frac"] > 0.9
        else:
            assert i1["sell_ptile_frac"] == 0.0 and i1["sell_constval_frac"] > 0.9
        assert i1["sell_ptile_frac"] <= i1["sell_constval_frac"]
        assert np.array_equal(_bits(y1), _bits(y0))
        _check(A, x, y1, bool(np.all(x == np.round(x))))


def test_ptile_misaligned_views_fall_back_bit_identical():
    """x / y one element into their buffers: not 16-byte aligned, so the
    bulk copies cannot run; the call takes the register path — same bits."""
    A = gen.laplacian2d(2048)
    x = gen.vector(5, gen.REAL, A.ncols)
    for compress in (True, False):
        ya, ia = _y(A, x, compress)
        for shift in (1, 2):
            yb, _ = _y(A, x, compress, shift=shift)
            assert np.array_equal(_bits(ya), _bits(yb)), (compress, shift)
        assert ia["sell_ptile_frac"] > 0.5
        _check(A, x, ya, False)


def _grid3(nz, ny, nx, offsets, center, off_val):
    """Constant-coefficient stencil on an nz x ny x nx grid (x fastest;
    Dirichlet: absent neighbours dropped), rows in CSR column order."""
    N = nz * ny * nx
    idx = np.arange(N)
    z, yv, xv = idx // (ny * nx), (idx // nx) % ny, idx % nx
    entries = []
    for dz, dy, dx in offsets:
        ok = (z + dz >= 0) & (z + dz < nz) & (yv + dy >= 0) & (yv + dy < ny) & (xv + dx >= 0) & (xv + dx < nx)
        entries.append((dz * ny * nx + dy * nx + dx, ok, center if (dz, dy, dx) == (0, 0, 0) else off_val))
    entries.sort(key=lambda e: e[0])
    per_row = np.zeros(N, np.int64)
    for _, ok, _ in entries:
        per_row += ok
    rp = np.concatenate([[0], np.cumsum(per_row)]).astype(np.int64)
    col = np.empty(rp[-1], np.int32)
    val = np.empty(rp[-1], np.float64)
    pos = rp[:-1].copy()
    for delta, ok, v in entries:
        r = idx[ok]
        col[pos[r]] = r + delta
        val[pos[r]] = v
        pos[r] += 1
    return gen.CSR(N, N, rp, col, val, 0, N)


@pytest.mark.parametrize("name", ["grid3d_7pt", "grid_8pt", "lap1d", "edge"])
def test_ptile_stencils(name):
    """A 3-D 7-point stencil on a 4 x 4 x 65536 grid (x-lines of 2046 interior
    chunks: 5 offset clusters ±nx·ny, ±nx, {-1, 0, 1} in single-line tiles —
    its lines would be too long for multi-line ones); a 3x3 stencil minus a
    corner (3 clusters of 2-3 offsets) on a 2048² grid; a 1-D 3-point stencil;
    and `edge`: 1600 rows with columns i+1..i+3 of 1603, one run of 50 chunks
    whose rounded range would end at x[1604]: its last chunk is trimmed off
    into the phase-A list (exactly 49 of 50 chunks tiled) — all
    bit-identical to the streamed layout and to the register path."""
    if name == "grid3d_7pt":
        offs = [(0, 0, 0), (-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]
        A = _grid3(4, 4, 65536, offs, 6.0, -1.0)
    elif name == "grid_8pt":
        offs = [(a, b) for a in (-1, 0, 1) for b in (-1, 0, 1) if (a, b) != (1, 1)]
        A = _stencil_grid(2048, offs, 8.0, -1.0)
    elif name == "lap1d":
        A = _stencil_grid(200_003, [(-1,), (0,), (1,)], 2.0, -1.0, dims=1)
    else:
        n = 1600
        col = (np.arange(n)[:, None] + np.array([1, 2, 3])[None, :]).ravel().astype(np.int32)
        val = np.tile(np.array([-1.0, 2.0, -1.0]), n)
        A = gen.CSR(n, n + 3, np.arange(0, 3 * n + 1, 3, dtype=np.int64), col, val, 0, n)
    for x in (gen.vector(3, gen.INT8, A.ncols), gen.vector(4, gen.REAL, A.ncols)):
        y1, i1 = _y(A, x, True)
        y0, _ = _y(A, x, False)
        y2, _ = _y(A, x, False, shift=1)   # register stencil-list path
        assert np.array_equal(_bits(y0), _bits(y2))
        if name == "edge":
            assert i1["sell_ptile_frac"] == pytest.approx(49 / 50)
        else:
            assert i1["sell_ptile_frac"] > 0.5
        assert np.array_equal(_bits(y1), _bits(y0))
        _check(A, x, y1, bool(np.all(x == np.round(x))))


@pytest.mark.parametrize("name", ["lap3d_96", "lap2d_300"])
def test_short_runs_keep_the_register_path(name):
    """Stencils whose runs are short (a 96³ grid: 1 interior chunk per x-line;
    a 300² grid: chunks straddle grid rows) get no tiles — they measured up to
    2.3x slower than the register paths — and stay bit-identical."""
    if name == "lap3d_96":
        offs = [(0, 0, 0), (-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]
        A = _stencil_grid(96, offs, 6.0, -1.0, dims=3)
    else:
        A = gen.laplacian2d(300)
    x = gen.vector(3, gen.INT8, A.ncols)
    y1, i1 = _y(A, x, True)
    y0, i0 = _y(A, x, False)
    assert i1["sell_ptile_frac"] == 0.0 and i0["sell_ptile_frac"] == 0.0
    assert np.array_equal(_bits(y1), _bits(y0))
    _check(A, x, y1, True)


def test_ptile_fp32_bit_identical_and_within_bound():
    A = gen.laplacian2d(2048)
    x = gen.vector(8, gen.REAL, A.ncols).astype(np.float32)
    A32 = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows)
    y1, i1 = _y(A32, x, True, dt=torch.float32)
    y0, i0 = _y(A32, x, False, dt=torch.float32)
    assert i1["sell_ptile_frac"] > 0.9 and i0["sell_ptile_frac"] > 0.9
    y2, _ = _y(A32, x, False, dt=torch.float32, shift=1)   # register stencil-list path
    assert np.array_equal(_bits(y0), _bits(y2))
    assert np.array_equal(_bits(y1), _bits(y0))
    b = oracle.bound_f32(A32, x)
    yr = oracle.spmv_f32(A32, x)
    assert np.all(np.abs(y1.astype(np.float64) - yr.astype(np.float64)) <= b)


def test_ptile_nonfinite_x():
    """Inf / NaN in x reach exactly the rows whose stencil touches them."""
    A = gen.laplacian2d(2048)
    x = gen.vector(9, gen.REAL, A.ncols)
    x[[5, 40_000, 2_131_000]] = [np.inf, np.nan, -np.inf]
    y1, _ = _y(A, x, True)
    y0, _ = _y(A, x, False)
    assert np.array_equal(_bits(y1), _bits(y0))
    yr = oracle.spmv(A, x)
    assert np.array_equal(np.isnan(y1), np.isnan(yr)) and np.array_equal(np.isinf(y1), np.isinf(yr))


def test_tile_plans_with_different_stage_sizes_interleave():
    """The kernel's dynamic shared-memory limit is a per-kernel attribute:
    a plan with smaller tiles created after one with larger tiles must not
    make the first plan's launches fail (4-rank distribution hang, round 2)."""
    A = gen.laplacian2d(2048)                                     # multi-line pattern tiles (5 lines / stage)
    B = _stencil_grid(300_000, [(-1,), (0,), (1,)], 2.0, -1.0, dims=1)   # one cluster: a small stage
    xa, xb = gen.vector(3, gen.INT8, A.ncols), gen.vector(4, gen.INT8, B.ncols)
    with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL) as pa, \
            pepp.Plan.from_csr(B, variant_mask=1 << pepp.V_SELL) as pb:
        ya = torch.full((A.nrows,), float("nan"), dtype=torch.float64, device="cuda")
        yb = torch.full((B.nrows,), float("nan"), dtype=torch.float64, device="cuda")
        for _ in range(3):
            pa.exec(torch.from_numpy(xa).cuda(), ya)
            pb.exec(torch.from_numpy(xb).cuda(), yb)
        torch.cuda.synchronize()
        assert pa.info()["sell_ptile_frac"] > 0.9 and pb.info()["sell_ptile_frac"] > 0.9
        assert np.array_equal(ya.cpu().numpy(), oracle.spmv(A, xa))
        assert np.array_equal(yb.cpu().numpy(), oracle.spmv(B, xb))


@pytest.mark.parametrize("name", ["lap2d", "eight_point"])
def test_multiline_pattern_tiles(name):
    """Grid stencils whose rows align with the chunks (grid line a multiple
    of 32) become multi-line pattern tiles — 5-point (W = 2), a 3x3 stencil
    minus a corner (clusters of 3, 3 and 2 offsets): the plan
    reports them, and y is bit-identical to the streamed layout and to the
    oracle."""
    if name == "lap2d":
        A = gen.laplacian2d(2048)
    else:
        offs = [(a, b) for a in (-1, 0, 1) for b in (-1, 0, 1) if (a, b) != (1, 1)]
        A = _stencil_grid(2048, offs, 8.0, -1.0)
    x = gen.vector(3, gen.INT8, A.ncols)
    y1, i1 = _y(A, x, True)
    y0, _ = _y(A, x, False)
    assert i1["sell_tile_multiline"] > 0, i1
    assert np.array_equal(_bits(y1), _bits(y0))
    _check(A, x, y1, True)
    xr = gen.vector(4, gen.REAL, A.ncols)
    y1, _ = _y(A, xr, True)
    y2, _ = _y(A, xr, True, shift=1)   # register path
    assert np.array_equal(_bits(y1), _bits(y2))


def test_nine_point_value_compression_multiline():
    """A 9-slot constant stencil (3x3) is a pattern-table entry (up to 16
    slots): value-compressed, multi-line tiles, bit-identical to the streamed
    layout and to the oracle."""
    offs = [(a, b) for a in (-1, 0, 1) for b in (-1, 0, 1)]
    A = _stencil_grid(2048, offs, 8.0, -1.0)
    x = gen.vector(3, gen.INT8, A.ncols)
    y1, i1 = _y(A, x, True)
    y0, i0 = _y(A, x, False)
    assert i1["sell_constval_frac"] > 0.9 and i1["sell_tile_multiline"] > 0 and i0["sell_constval_frac"] == 0.0
    assert np.array_equal(_bits(y1), _bits(y0))
    _check(A, x, y1, True)


def test_few_tiles_many_general_chunks():
    """A plan whose pattern tiles are only part of the matrix (the first 60 %
    of the rows a constant 3-point stencil, the rest random columns): the
    chunks outside the tiles are walked by the full-grid SELL kernel beside
    the tile kernel (two launches), not by its few walker warps (a plan with
    250 tiled and 524 K general chunks took 34.8 ms through them); y equals
    the oracle."""
    n = 1 << 20
    cut = (n * 6 // 10) // 32 * 32
    S = _stencil_grid(cut, [(-1,), (0,), (1,)], 2.0, -1.0, dims=1)
    U = gen.uniform(n - cut, n, 16, seed=12, val_mode=gen.INT4)
    rp = np.concatenate([S.row_ptr[:-1], U.row_ptr + S.row_ptr[-1]]).astype(np.int64)
    C = gen.CSR(n, n, rp, np.concatenate([S.col, U.col]).astype(np.int32), np.concatenate([S.val, U.val]), 0, n)
    x = gen.vector(5, gen.INT8, C.ncols)
    with pepp.Plan.from_csr(C, variant_mask=1 << pepp.V_SELL) as plan:
        xd = torch.from_numpy(x).cuda()
        y = torch.full((C.nrows,), float("nan"), dtype=torch.float64, device="cuda")
        for _ in range(3):
            u = plan.exec(xd, y)
        torch.cuda.synchronize()
        info = plan.info()
        assert 0.5 < info["sell_ptile_frac"] < 0.7, info
        assert u.launches == 2
        assert np.array_equal(y.cpu().numpy(), oracle.spmv(C, x))


def test_minority_constant_chunks_keep_the_stencil_list():
    """Value compression only where it covers most chunks: a random-valued
    band with a constant block (125 of 32 K chunks) keeps every stencil chunk
    on the stencil list — stencil tiles, one launch — instead of sending the
    band through the general walk; y equals the oracle."""
    B = gen.banded(1 << 20, 4, seed=11, val_mode=gen.INT4)
    rp = np.asarray(B.row_ptr)
    val = B.val.copy()
    for r in range(64, 4096):                       # a constant 9-point block: 125 full chunks
        s, e = int(rp[r]), int(rp[r + 1])
        val[s:e] = np.where(B.col[s:e] == r, 8.0, -1.0)
    C = gen.CSR(B.nrows, B.ncols, B.row_ptr, B.col, val, 0, B.nrows)
    x = gen.vector(5, gen.INT8, C.ncols)
    with pepp.Plan.from_csr(C, variant_mask=1 << pepp.V_SELL) as plan:
        xd = torch.from_numpy(x).cuda()
        y = torch.full((C.nrows,), float("nan"), dtype=torch.float64, device="cuda")
        for _ in range(3):
            u = plan.exec(xd, y)
        torch.cuda.synchronize()
        info = plan.info()
        assert info["sell_constval_frac"] == 0.0 and info["sell_ptile_frac"] > 0.9, info
        assert u.launches == 1
        assert np.array_equal(y.cpu().numpy(), oracle.spmv(C, x))
