"""Column panels vs the row-major variants on uniform random 16/row matrices
whose x leaves L2 (config 5's random sweep points >= 10^7 rows): every
candidate forced (median of back-to-back calls, device events), the
calibrated automatic choice, and the plan time."""
import json
import os
import statistics
import sys
import time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
import gen
import paper_conf_sc_dastgeerlk12_b200 as pepp

sizes = [int(float(a)) for a in sys.argv[1:]] or [10_000_000, 31_622_777, 100_000_000]
for n in sizes:
    A = gen.uniform(n, n, 16, seed=100 + n % 97)
    x = torch.from_numpy(gen.vector(7, gen.REAL, n)).cuda()
    y = torch.empty(n, dtype=torch.float64, device="cuda")
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    plan = pepp.Plan.from_csr(A)
    torch.cuda.synchronize()
    plan_s = time.perf_counter() - t0
    del A
    res = {"rows": n, "plan_s": round(plan_s, 2), "device_gb": round(plan.info()["device_bytes"] / 1e9, 1)}
    only = os.environ.get("PANEL_ONLY")
    for c in plan.candidates():
        if only and c.variant != pepp.V_PANEL:
            continue
        f = pepp.Choice(c.variant, c.param)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(6)]
        for a, b in ev:
            a.record()
            plan.exec(x, y, force=f)
            b.record()
        torch.cuda.synchronize()
        res[c.name] = round(statistics.median(a.elapsed_time(b) for a, b in ev[1:]) * 1e3, 1)
    for _ in range(60):
        u = plan.exec(x, y)
    torch.cuda.synchronize()
    res["auto"] = plan.select().name
    print(json.dumps(res), flush=True)
    plan.close()
    del x, y
    torch.cuda.empty_cache()
