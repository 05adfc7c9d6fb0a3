"""Library cross-check: cuSPARSE's CSR SpMV (through
torch.sparse_csr_tensor) on the same inputs agrees with the oracle within the
north-star bound, and so does every variant of ours — three implementations
that share nothing (plain C oracle, NVIDIA's library, our kernels). Extra
confidence for the oracle on GPU-sized real-valued inputs; not a parity source."""
from __future__ import annotations

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _cusparse(A, x):
    crow = torch.from_numpy(A.row_ptr - A.row_ptr[0]).cuda().to(torch.int32)
    col = torch.from_numpy(A.col).cuda().to(torch.int32)
    val = torch.from_numpy(A.val).cuda()
    M = torch.sparse_csr_tensor(crow, col, val, size=(A.nrows, A.ncols))
    return (M @ torch.from_numpy(x).cuda()).cpu().numpy()


@pytest.mark.parametrize("name", ["uniform", "zipf", "lap"])
def test_cusparse_oracle_ours_agree(name):
    import gen
    import oracle
    import paper_conf_sc_dastgeerlk12_b200 as pepp
    A = {"uniform": lambda: gen.uniform(200_000, 200_000, 16, seed=42),
         "zipf": lambda: gen.zipf(100_000, 100_000, seed=46),
         "lap": lambda: gen.laplacian2d(300)}[name]()
    x = gen.vector(45, gen.REAL, A.ncols)
    ref = oracle.spmv(A, x)
    tol = oracle.bound(A, x)
    yl = _cusparse(A, x)
    assert np.all(np.abs(yl - ref) <= tol), "cuSPARSE outside the bound of the oracle"
    with pepp.Plan.from_csr(A, prune=False) as plan:
        xd = torch.from_numpy(x).cuda()
        y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
        for c in plan.candidates():
            plan.exec(xd, y, force=pepp.Choice(c.variant, c.param))
            torch.cuda.synchronize()
            yo = y.cpu().numpy()
            assert np.all(np.abs(yo - ref) <= tol), c.name
            assert np.all(np.abs(yo - yl) <= 2 * tol), c.name   # both within the bound of the exact sum
