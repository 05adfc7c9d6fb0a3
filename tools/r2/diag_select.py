"""Selector diagnostics on config 4 (bench.py's plan options): after the
bench's warm-up (3 steps of 100 iterated calls), print every candidate's
history count / mean / stddev and the calls' choices."""
import json
import math
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch
import gen
import paper_conf_sc_dastgeerlk12_b200 as pepp

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A = gen.laplacian2d(n)
x0 = gen.vector(4, gen.REAL, A.ncols)
plan = pepp.Plan.from_csr(A, compress_values=False)
st = torch.cuda.Stream()
xs = torch.from_numpy(x0).cuda()
bufs = [torch.empty(A.nrows, dtype=torch.float64, device="cuda") for _ in range(2)]
seq = []
for step in range(4):
    with torch.cuda.stream(st):
        src = xs
        for k in range(100):
            u = plan.exec(src, bufs[k & 1], flags=pepp.Y_LOCAL, stream=st)
            seq.append((u.name, u.calibrating))
            src = bufs[k & 1]
    st.synchronize()
plan.flush_history()
out = {"first_calls": seq[:60], "last": seq[-1]}
for i, c in enumerate(plan.candidates()):
    cnt, mean, m2 = plan.history_stats(i)
    out[c.name] = (cnt, round(mean, 1), round(math.sqrt(m2 / max(1, cnt - 1)), 1))
print(json.dumps(out))
plan.close()
