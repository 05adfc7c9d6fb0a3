"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (its plan options — compress_values = 0, the headline — and the
library default compress_values = 1, in fp64 and the fp32 instance;
automatic per-call selection), on sampled rows the oracle computes one by one
(SURVEY.md §8(c) P5/P6/P7):

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


LAYOUTS = [pytest.param(False, "f64", id="values_streamed-f64"),    # bench.py's headline plan
           pytest.param(True, "f64", id="value_compressed-f64"),    # the library default
           pytest.param(False, "f32", id="values_streamed-f32"),    # bench.py --dtype f32
           pytest.param(True, "f32", id="value_compressed-f32")]


def _typed(A, dt):
    return A if dt == "f64" else gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0,
                                         A.global_nrows)


@pytest.mark.parametrize("compress,dt", LAYOUTS)
def test_config4_integer_iterations_bitwise_on_sampled_rows(lap8192, compress, dt):
    """bench.py's plan options (compress_values = 0: the fp64 / fp32
    stencil-list kernel + the genlist walk; = 1: the pattern-table layout),
    automatic selection, iterated; integer x0: every sampled row of x_k equals
    the oracle applied to the GPU's own x_{k-1}, bit for bit (k = 1 and the
    last step; fp32 stops at k = 6, where |x| < 2^24 keeps float exact)."""
    A = lap8192
    n = 8192
    R = A.nrows
    K = 16 if dt == "f64" else 6
    tdt = torch.float64 if dt == "f64" else torch.float32
    rows = _sample_rows(R, extra=[n - 1, n, R - n - 1, R - n, R // 2, 32 * 4000 + 31, 32 * 4001])
    x0 = gen.vector(3, gen.INT8, R)
    with pepp.Plan.from_csr(_typed(A, dt), compress_values=compress) as plan:
        info = plan.info()
        if compress:
            assert info["sell_constval_frac"] > 0.9
        else:
            assert info["sell_constval_frac"] == 0 and info["sell_stencil_frac"] > 0.9
        a = torch.from_numpy(x0).to(tdt).cuda()
        b = torch.empty_like(a)
        c = torch.empty_like(a)
        for _ in range(40):   # calibration first, as in bench.py's warm-up: then the timed choice runs
            plan.exec(a, c, flags=pepp.Y_NEXT_INPUT)
        used = plan.exec(a, b, flags=pepp.Y_NEXT_INPUT)
        torch.cuda.synchronize()
        x1 = b.cpu().numpy().astype(np.float64)
        assert np.array_equal(x1[rows], oracle.spmv_rows(A, x0, rows)), used.name
        src, dst = b, c
        names = set()
        for _ in range(K - 2):
            names.add(plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT).name)
            src, dst = dst, src
        torch.cuda.synchronize()
        xp = src.cpu().numpy().astype(np.float64)
        u = plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
        torch.cuda.synchronize()
        xK = dst.cpu().numpy().astype(np.float64)
    assert np.abs(xK).max() < (2.0 ** 53 if dt == "f64" else 2.0 ** 24)
    assert np.array_equal(xK[rows], oracle.spmv_rows(A, xp, rows)), (u.name, names)
    assert names | {u.name, used.name} == {"sell[1]"}   # the SELL layout under test is what ran


@pytest.mark.parametrize("compress,dt", LAYOUTS)
def test_config4_real_iterations_single_steps_within_bound(lap8192, compress, dt):
    """100 iterations from a real x0 (bench.py's workload), single steps
    k = 1, 50, 100 within the per-row bound of the oracle applied to the GPU's
    own x_{k-1}: fp64 2·n·2^-52·Σ|a||x|; fp32 2·n·2^-23·Σ|a||x| against the
    fp64 oracle on the same float inputs (which is within n·2^-53·Σ|a||x| of
    the exact sum, far inside)."""
    A = lap8192
    R = A.nrows
    rows = _sample_rows(R, seed=1)
    tdt = torch.float64 if dt == "f64" else torch.float32
    x0 = gen.vector(4, gen.REAL, R)
    if dt == "f32":
        x0 = x0.astype(np.float32).astype(np.float64)
    check = {1, 50, 100}
    with pepp.Plan.from_csr(_typed(A, dt), compress_values=compress) as plan:
        bufs = [torch.from_numpy(x0).to(tdt).cuda(), torch.empty(R, dtype=tdt, device="cuda"),
                torch.empty(R, dtype=tdt, device="cuda")]
        src = bufs[0]
        for _ in range(40):   # calibration first (bench.py's warm-up)
            plan.exec(bufs[0], bufs[2], flags=pepp.Y_NEXT_INPUT)
        prev_host = x0
        for k in range(1, 101):
            dst = bufs[1] if src is not bufs[1] else bufs[2]
            used = plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
            if k in check:
                torch.cuda.synchronize()
                xk = dst.cpu().numpy().astype(np.float64)
                ref = oracle.spmv_rows(A, prev_host, rows)
                bnd = oracle.bound_rows(A, prev_host, rows)
                if dt == "f32":
                    bnd = np.ldexp(bnd, 29)       # 2·n·2^-52·S -> 2·n·2^-23·S
                assert oracle.within(xk[rows], ref, bnd).all(), (k, used.name)
                assert used.name == "sell[1]"
            if k + 1 in check:
                torch.cuda.synchronize()
                prev_host = dst.cpu().numpy().astype(np.float64)
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
