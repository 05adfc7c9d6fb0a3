"""Where pepp_spmv_plan's time goes on config 4: the plan built with one
variant at a time (validation + copy always), pageable vs pinned host arrays."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, gen
import paper_conf_sc_dastgeerlk12_b200 as pepp
A = gen.laplacian2d(8192)
torch.cuda.synchronize()
res = {}
def t(name, **kw):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    p = pepp.Plan.from_csr(A, **kw); torch.cuda.synchronize()
    res[name] = round((time.perf_counter() - t0) * 1e3, 1)
    p.close(); torch.cuda.empty_cache()
t("warm", variant_mask=1 << pepp.V_CSR_VECTOR)
for nm, v in [("csr_vector", pepp.V_CSR_VECTOR), ("merge_path", pepp.V_MERGE_PATH), ("sell", pepp.V_SELL),
              ("csr_stream", pepp.V_CSR_STREAM)]:
    t(nm, variant_mask=1 << v)
t("all", variant_mask=0)
t("all_compress0", variant_mask=0, compress_values=False)
t("sell_novalidate", variant_mask=1 << pepp.V_SELL, validate=False)
print(json.dumps(res))
res2 = {}
for nm, kw in [("sell_c1", dict(variant_mask=1 << pepp.V_SELL, compress_values=True)),
               ("sell_c0", dict(variant_mask=1 << pepp.V_SELL, compress_values=False)),
               ("sell_c1_again", dict(variant_mask=1 << pepp.V_SELL, compress_values=True))]:
    torch.cuda.synchronize(); t0 = time.perf_counter()
    p = pepp.Plan.from_csr(A, **kw); torch.cuda.synchronize()
    res2[nm] = round((time.perf_counter() - t0) * 1e3, 1)
    p.close()
print(json.dumps(res2))
