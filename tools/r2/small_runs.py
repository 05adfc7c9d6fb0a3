"""Tile path vs register path (x / y one element off) on stencils whose
tile runs are short: 3-D 7-point grids with x-lines of 96 / 160 / 256 rows
(runs of 1 / 3 / 6 chunks), both layouts."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch, gen
import paper_conf_sc_dastgeerlk12_b200 as pepp
from test_gpu_parity import _stencil_grid

def timed(plan, x, y, reps=20):
    for _ in range(5): plan.exec(x, y)
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in ev:
        a.record(); plan.exec(x, y); b.record()
    torch.cuda.synchronize()
    return round(float(np.median([a.elapsed_time(b) for a, b in ev])) * 1e3, 2)

offs = [(0, 0, 0), (-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]
for n in [int(v) for v in (sys.argv[1:] or ["96", "160", "256"])]:
    A = _stencil_grid(n, offs, 6.0, -1.0, dims=3)
    for cz in (True, False):
        with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, compress_values=cz) as plan:
            xb = torch.zeros(A.ncols + 1, dtype=torch.float64, device="cuda"); xb[1:] = torch.from_numpy(gen.vector(4, gen.REAL, A.ncols)).cuda()
            yb = torch.empty(A.nrows + 1, dtype=torch.float64, device="cuda")
            t_tile = timed(plan, xb[1:].clone(), yb[1:].clone())
            t_reg = timed(plan, xb[1:], yb[1:])
            i = plan.info()
            print(json.dumps({"n": n, "rows": A.nrows, "compress": cz, "tile_us": t_tile, "register_us": t_reg,
                              "tile_frac": i["sell_ptile_frac"], "multiline": i["sell_tile_multiline"]}), flush=True)
