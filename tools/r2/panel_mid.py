"""Uniform random 16/row matrices with x between 32 and 96 MB (4e6 .. 1.2e7
rows): every candidate forced, median µs with an L2 flush between calls —
does the column-panel layout pay below the 96 MB threshold?"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen
import paper_conf_sc_dastgeerlk12_b200 as pepp
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for n in [int(v) for v in (sys.argv[1:] or ["4000000", "6000000", "10000000", "12000000"])]:
    A = gen.uniform(n, n, 16, seed=7)
    x = torch.from_numpy(gen.vector(8, gen.REAL, n)).cuda()
    y = torch.empty(n, dtype=torch.float64, device="cuda")
    with pepp.Plan.from_csr(A) as plan:
        res = {}
        for c in plan.candidates():
            f = pepp.Choice(c.variant, c.param)
            for _ in range(2): plan.exec(x, y, force=f)
            ts = []
            for _ in range(9):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(); u = plan.exec(x, y, force=f); e1.record(); torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e3)
            res[u.name] = round(float(np.median(ts)), 1)
        print(json.dumps({"rows": n, "x_mb": n * 8 / 2**20, "us": res}), flush=True)
