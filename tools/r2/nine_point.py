"""9-point constant-coefficient stencil (2-D, 4096^2 rows): the SELL layout
with value compression (pattern table up to 16 slots) vs values streamed,
plus config 4 value-compressed through the aligned tile path and through the
register fallback (x / y views one element off)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
import numpy as np, torch, gen
import paper_conf_sc_dastgeerlk12_b200 as pepp
from test_gpu_parity import _stencil_grid

def timed(plan, x, y, reps=30):
    for _ in range(5): plan.exec(x, y)
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in ev:
        a.record(); u = plan.exec(x, y); b.record()
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(b) for a, b in ev])) * 1e3, u

offs = [(a, b) for a in (-1, 0, 1) for b in (-1, 0, 1)]
A = _stencil_grid(4096, offs, 8.0, -1.0)
for cz in (True, False):
    with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, compress_values=cz) as plan:
        x = torch.from_numpy(gen.vector(4, gen.REAL, A.ncols)).cuda(); y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
        us, u = timed(plan, x, y)
        i = plan.info()
        print(json.dumps({"matrix": "9pt 4096^2", "compress": cz, "us": round(us, 2), "layout_bytes": u.layout_bytes,
                          "constval_frac": i["sell_constval_frac"], "tile_frac": i["sell_ptile_frac"],
                          "multiline": i["sell_tile_multiline"]}), flush=True)
A = gen.laplacian2d(8192)
with pepp.Plan.from_csr(A, variant_mask=1 << pepp.V_SELL, compress_values=True) as plan:
    xb = torch.zeros(A.ncols + 1, dtype=torch.float64, device="cuda"); xb[1:] = torch.from_numpy(gen.vector(4, gen.REAL, A.ncols)).cuda()
    yb = torch.empty(A.nrows + 1, dtype=torch.float64, device="cuda")
    for nm, (x, y) in {"aligned": (xb[1:].clone(), yb[1:].clone()), "misaligned": (xb[1:], yb[1:])}.items():
        us, u = timed(plan, x, y, 20)
        print(json.dumps({"matrix": "lap8192 vc", "path": nm, "us": round(us, 2), "launches": u.launches}), flush=True)
