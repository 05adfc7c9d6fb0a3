#!/usr/bin/env python3
"""Host-side cost per call (no GPU work in the way: a 4 K-row matrix):
pepp_spmv_select through ctypes, pepp_spmv_exec through ctypes with
prebuilt arguments (the library's own cost + one kernel launch), and
Plan.exec (the binding's marshalling on top). Prints one JSON line per matrix.

  python tools/select_overhead.py
"""
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402


def per_call(fn, n):
    for _ in range(200):
        fn()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(n):
        fn()
    host = (time.perf_counter() - t) / n * 1e6
    torch.cuda.synchronize()
    return round(host, 3), round((time.perf_counter() - t) / n * 1e6, 3)


for A in (gen.laplacian2d(64), gen.uniform(100000, 100000, 16, seed=1)):
    with pepp.Plan.from_csr(A, prune=False) as plan:
        x = torch.zeros(A.ncols, dtype=torch.float64, device="cuda")
        y = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
        for _ in range(400):
            if not plan.exec(x, y).calibrating:
                break
        plan.flush_history()
        L = pepp._capi.lib()
        c = pepp._capi.CHOICE_T()
        ref, h = ctypes.byref(c), plan._h
        st = torch.cuda.current_stream().cuda_stream
        px, py = x.data_ptr(), y.data_ptr()
        sel = per_call(lambda: L.pepp_spmv_select(h, ref), 20000)[0]
        cexec = per_call(lambda: L.pepp_spmv_exec(h, px, py, 0, st, None, ref), 5000)
        pyexec = per_call(lambda: plan.exec(x, y), 5000)
        print(json.dumps({"matrix": A.name, "select_us": sel, "c_exec_host_us": cexec[0], "c_exec_incl_gpu_us": cexec[1],
                          "py_exec_host_us": pyexec[0], "py_exec_incl_gpu_us": pyexec[1]}), flush=True)
