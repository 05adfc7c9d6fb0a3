"""Tile path vs register path (x / y views one element off) on 2-D Laplacians
of several widths and 3-D 7-point grids: where do the tiles pay? Prints the
mean rows per tile beside the times (both layouts)."""
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

cases = [("2d", n) for n in (256, 512, 1024, 2048, 4096)] + [("3d", n) for n in (128, 192, 320)]
offs3 = [(0, 0, 0), (-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]
for kind, n in cases:
    A = gen.laplacian2d(n) if kind == "2d" else _stencil_grid(n, offs3, 6.0, -1.0, dims=3)
    for cz in (True, False):
        with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, compress_values=cz) as plan:
            xb = torch.zeros(A.ncols + 1, dtype=torch.float64, device="cuda"); xb[1:] = torch.from_numpy(gen.vector(4, gen.REAL, A.ncols)).cuda()
            yb = torch.empty(A.nrows + 1, dtype=torch.float64, device="cuda")
            t_tile = timed(plan, xb[1:].clone(), yb[1:].clone())
            t_reg = timed(plan, xb[1:], yb[1:])
            i = plan.info()
            print(json.dumps({"kind": kind, "n": n, "rows": A.nrows, "compress": cz, "tile_us": t_tile, "register_us": t_reg,
                              "ratio": round(t_tile / t_reg, 3), "tile_frac": round(i["sell_ptile_frac"], 3)}), flush=True)
