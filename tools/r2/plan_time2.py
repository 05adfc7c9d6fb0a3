import json, os, sys, time
sys.path.insert(0, os.getcwd())
import torch, gen, paper_conf_sc_dastgeerlk12_b200 as pepp
A = gen.laplacian2d(8192)
res = []
for rep in range(2):
    for c in (True, False):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        p = pepp.Plan.from_csr(A, compress_values=c); torch.cuda.synchronize()
        res.append((c, round((time.perf_counter() - t0) * 1e3, 1)))
        p.close()
print(res)
