"""The fp32 instance (the paper's own `float` signature,
P@32944): every variant in fp32 against the fp32 oracle (fp32 products and
sums). Integer-valued inputs whose partial sums stay below 2^24 -> bit-exact;
real inputs -> per row |y - y_ref| <= 2·nnz_row·2^-23·Σ|a||x|."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402


def _f32(A):
    return gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows, A.name)


CASES = {
    "lap_int": lambda: (gen.laplacian2d(64), gen.vector(1, gen.INT8, 4096), True),
    "lap_real": lambda: (gen.laplacian2d(64), gen.vector(2, gen.REAL, 4096), False),
    "uniform_int": lambda: (gen.uniform(50_000, 50_000, 16, seed=43, val_mode=gen.INT4), gen.vector(44, gen.INT8, 50_000), True),
    "zipf_int": lambda: (gen.zipf(60_000, 60_000, seed=47, val_mode=gen.INT4), gen.vector(48, gen.INT8, 60_000), True),
    "zipf_real": lambda: (gen.zipf(60_000, 60_000, seed=46), gen.vector(49, gen.REAL, 60_000), False),
    "banded_real": lambda: (gen.banded(30_001, 4, seed=100), gen.vector(101, gen.REAL, 30_001), False),
}


def _run(plan, x, force=None):
    xd = torch.from_numpy(x).cuda()
    y = torch.full((plan.nrows,), float("nan"), dtype=torch.float32, device="cuda")
    used = plan.exec(xd, y, force=force)
    torch.cuda.synchronize()
    return y.cpu().numpy(), used


@pytest.mark.parametrize("compress", [True, False])
@pytest.mark.parametrize("case", sorted(CASES))
def test_every_variant_fp32(case, compress):
    """compress = False keeps stencil values streamed: the fp32 SELL plan then
    runs its stencil chunks through the stencil-list kernel (sell_slist_kernel)
    and the rest through the genlist walk."""
    A, x, exact = CASES[case]()
    A32, x32 = _f32(A), x.astype(np.float32)
    ref = oracle.spmv(A32, x32)
    assert ref.dtype == np.float32
    with pepp.Plan.from_csr(A32, prune=False, compress_values=compress) as plan:
        assert plan.value_type == pepp._capi.VALUE_F32
        forces = [pepp.Choice(c.variant, c.param) for c in plan.candidates()]
        assert {f.variant for f in forces} == {pepp.V_CSR_VECTOR, pepp.V_MERGE_PATH, pepp.V_SELL, pepp.V_CSR_STREAM}
        for f in forces:
            y, used = _run(plan, x32, f)
            assert y.dtype == np.float32
            if exact:
                assert np.array_equal(y, ref), used.name
            else:
                b = oracle.bound_f32(A32, x32)
                diff = np.abs(y.astype(np.float64) - ref.astype(np.float64))
                assert np.all(diff <= b), (used.name, np.flatnonzero(diff > b)[:5])
            if f.variant == pepp.V_CSR_STREAM:   # short rows: the oracle's fp32 arithmetic exactly
                short = np.diff(A.row_ptr) <= 64
                assert np.array_equal(y[short], ref[short])


def test_fp32_iterate_graph_and_host_path():
    n = 48
    A32 = _f32(gen.laplacian2d(n))
    x0 = gen.vector(3, gen.INT8, n * n).astype(np.float32)
    K = 5   # |x| stays below 2^24: exact
    ref = x0.copy()
    for _ in range(K):
        ref = oracle.spmv(A32, ref)
    with pepp.Plan.from_csr(A32) as plan:
        x = torch.from_numpy(x0).cuda()
        y = torch.empty_like(x)
        w = torch.empty_like(x)
        g = plan.graph(x, y, iterations=K, mode=1, work=w)
        g.launch()
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy(), ref)   # K odd: result in y
        g.close()
        yh = np.empty(n * n, dtype=np.float32)
        plan.exec_host(x0, yh, iterations=K)
        assert np.array_equal(yh, ref)
        # containers hold fp64: an fp32 plan refuses them
        v, u = pepp.Vector(n * n), pepp.Vector(n * n)
        with pytest.raises(pepp.PeppError) as e:
            plan.exec_vec(v, u)
        assert e.value.status == pepp._capi.PEPP_E_UNSUPPORTED


def test_fp32_differs_from_fp64_where_float_rounds():
    """The fp32 path really computes in float: 1 + 2^-24 + 2^-24 stays 1."""
    A = gen.CSR(1, 3, np.array([0, 3], np.int64), np.array([0, 1, 2], np.int32), np.ones(3, np.float32), 0, 1)
    x = np.array([1.0, 2.0 ** -24, 2.0 ** -24], dtype=np.float32)
    with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_CSR_STREAM) as plan:
        y, _ = _run(plan, x)
    assert y[0] == np.float32(1.0) == oracle.spmv(A, x)[0]


def test_fp32_stencil_list_large_bitwise():
    """The fp32 stencil path at a size spanning many warps and the
    straddling groups between offset sets (a 1024² Laplacian has 3 stencil
    offset sets plus the general boundary chunks): integer inputs bit-exact;
    one launch (the tile kernel, its walker warps taking the boundary chunks)
    — two (stencil-list kernel + genlist walk) when x / y are not 16-byte
    aligned."""
    A = gen.laplacian2d(1024)
    A32 = _f32(A)
    x32 = gen.vector(7, gen.INT8, A.ncols).astype(np.float32)
    ref = oracle.spmv(A32, x32)
    with pepp.Plan.from_csr(A32, variant_mask=1 << pepp.V_SELL, compress_values=False) as plan:
        y, used = _run(plan, x32)
        assert used.launches == 1
        assert np.array_equal(y, ref)
        xo = torch.zeros(A.ncols + 1, dtype=torch.float32, device="cuda")
        xo[1:] = torch.from_numpy(x32).cuda()
        yo = torch.full((A.nrows + 1,), float("nan"), dtype=torch.float32, device="cuda")
        u = plan.exec(xo[1:], yo[1:])
        torch.cuda.synchronize()
        assert u.launches == 2 and np.array_equal(yo[1:].cpu().numpy(), ref)
        # the same path captured in a CUDA graph (the genlist walk's fork /
        # join onto the plan's second stream becomes a graph branch)
        xd = torch.from_numpy(x32).cuda()
        yd = torch.full((A.nrows,), float("nan"), dtype=torch.float32, device="cuda")
        g = plan.graph(xd, yd, iterations=3, mode=0)
        g.launch()
        torch.cuda.synchronize()
        g.close()
        assert np.array_equal(yd.cpu().numpy(), ref)
