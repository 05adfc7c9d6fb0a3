"""Time the SELL layout of Laplacians: average µs per SpMV over back-to-back
calls after calibration, the layout bytes and the fraction of the measured
copy peak. Arguments n:dtype[:compress] (compress 1 = opts.compress_values,
the library default; 0 = values streamed, the bench headline's layout)."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch
import gen
import paper_conf_sc_dastgeerlk12_b200 as pepp

peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6545.0
for arg in (sys.argv[1:] or ["8192:f64", "8192:f32", "4096:f64"]):
    n, dt, *cz = arg.split(":")
    n, cz = int(n), bool(int(cz[0])) if cz else True
    A = gen.laplacian2d(n)
    if dt == "f32":
        A = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows)
    tdt = torch.float32 if dt == "f32" else torch.float64
    plan = pepp.Plan.from_csr(A, compress_values=cz, variant_mask=1 << pepp.V_SELL)
    x = torch.from_numpy(gen.vector(4, gen.REAL, A.ncols)).to(tdt).cuda()
    ys = [torch.empty(A.nrows, dtype=tdt, device="cuda") for _ in range(2)]
    for k in range(20):
        plan.exec(x if k == 0 else ys[(k - 1) & 1], ys[k & 1])
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(50)]
    src = x
    for k, (a, b) in enumerate(ev):
        a.record()
        u = plan.exec(src, ys[k & 1])
        b.record()
        src = ys[k & 1]
    torch.cuda.synchronize()
    us = float(np.mean([a.elapsed_time(b) for a, b in ev])) * 1e3
    print(json.dumps({"n": n, "dtype": dt, "compress": int(cz), "us": round(us, 2), "layout_bytes": u.layout_bytes,
                      "frac": round(u.layout_bytes / (us * 1e-6) / 1e9 / peak, 4), "launches": u.launches,
                      "constval_frac": plan.info()["sell_constval_frac"],
                      "tile_frac": plan.info()["sell_ptile_frac"]}), flush=True)
    plan.close()
