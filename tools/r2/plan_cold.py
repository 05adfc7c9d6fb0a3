"""Plan time of the bench headline's plan (config 4, every variant, values
streamed) in a fresh process: first plan (pinned staging pool allocated) and
a second one."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch, gen
import paper_conf_sc_dastgeerlk12_b200 as pepp
torch.cuda.init(); torch.zeros(1, device="cuda")
A = gen.laplacian2d(8192)
out = {}
for k in range(2):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    p = pepp.Plan.from_csr(A, compress_values=False)
    torch.cuda.synchronize(); out[f"plan{k}_ms"] = round((time.perf_counter() - t0) * 1e3, 1)
    p.close()
print(json.dumps(out))
