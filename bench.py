#!/usr/bin/env python3
"""Benchmark of the SpMV hot path (BASELINE.json metric: SpMV GFLOP/s and
achieved HBM GB/s (% of HBM) at 1/2/4/8 B200).

Default workload = BASELINE.json config 4: 2D 5-point Laplacian on an
8192x8192 grid (67,108,864 rows, 335,511,552 nnz, fp64), 100 iterated SpMVs
x_{k+1} = A·x_k per step, rows nnz-balanced over N ranks (one process per
GPU), NCCL exchange of y between iterations. The matrix (5.4 GB of
algorithmic bytes per SpMV) is far larger than L2 (126 MB), so no flush is
needed between iterations. Every step goes through the C-ABI
(pepp_spmv_exec per iteration: per-call variant selection + kernel +
exchange + history update).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--workload lap8192|uniform1m|zipf4m|lap64] [--iters I] [--variant csr_vector:4|merge_path|sell]

One JSON line on rank 0. Multi-GPU: launched by torchrun (RANK / WORLD_SIZE /
LOCAL_RANK / MASTER_* from the environment), or `--gpus N` alone re-executes
itself under torch.distributed.run with N ranks; times are device events, max
over ranks. The default line also carries BASELINE configs 1-3 (`configs`:
per-SpMV time, layout-bytes roofline fraction, selector ratio, plan time,
cold single call with the matrix upload).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    "lap8192": dict(desc="BASELINE config 4: 2D 5-point Laplacian 8192x8192 (67.1M rows, 335.5M nnz), fp64, "
                         "100 iterated SpMVs per step, nnz-balanced row blocks over N GPUs, NCCL exchange",
                    iters=100, iterated=True),
    "uniform1m": dict(desc="BASELINE config 2: uniform random 1M x 1M, 16 nnz/row (16.8M nnz), fp64",
                      iters=20, iterated=False),
    "zipf4m": dict(desc="BASELINE config 3: power-law rows P(k)~k^-1.5, k<=435, 4M x 4M (~67M nnz), fp64",
                   iters=20, iterated=False),
    "lap64": dict(desc="BASELINE config 1: 2D 5-point Laplacian 64x64 (4096 rows, 20224 nnz), fp64",
                  iters=1000, iterated=False),
    "lap2048": dict(desc="test-sized Laplacian 2048x2048 (4.2M rows), iterated like config 4 (not a BASELINE config)",
                    iters=100, iterated=True),
    "skew": dict(desc="heavy-tailed rows (not a BASELINE config): P(k)~k^-2, k<=4M, 4M x 4M, fp64 — rows up to ~1e6 nnz",
                 iters=20, iterated=False),
}


# --------------------------------------------------------------- inputs
def make_block(workload: str, r0: int, r1: int):
    import gen
    if workload == "lap8192":
        return gen.laplacian2d(8192, r0, r1)
    if workload == "lap64":
        return gen.laplacian2d(64, r0, r1)
    if workload == "lap2048":
        return gen.laplacian2d(2048, r0, r1)
    if workload == "uniform1m":
        return gen.uniform(1 << 20, 1 << 20, 16, seed=42, r0=r0, r1=r1)
    if workload == "zipf4m":
        return gen.zipf(4 << 20, 4 << 20, seed=46, r0=r0, r1=r1)
    if workload == "skew":
        return gen.zipf(4 << 20, 4 << 20, seed=50, alpha=2.0, kmax=4 << 20, r0=r0, r1=r1)
    raise ValueError(workload)


def global_rowptr(workload: str) -> np.ndarray:
    import ctypes

    import gen
    if workload in ("lap8192", "lap64", "lap2048"):
        n = {"lap8192": 8192, "lap64": 64, "lap2048": 2048}[workload]
        rp = np.empty(n * n + 1, dtype=np.int64)
        gen.lib().gen_laplacian2d_rowptr(n, 0, n * n, rp.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)))
        return rp
    if workload == "uniform1m":
        return np.arange(0, ((1 << 20) + 1) * 16, 16, dtype=np.int64)
    if workload == "skew":
        return gen._rowptr_global(1, 50, 4 << 20, 4 << 20, 2.0, 4 << 20, 0, 4 << 20)
    return gen._rowptr_global(1, 46, 4 << 20, 4 << 20, 1.5, 435, 0, 4 << 20)


def x0_vector(workload: str, n: int) -> np.ndarray:
    import gen
    return gen.vector(4, gen.REAL, n)   # real x0 ~ U[-1,1) (config 4's real mode, seed 4)


# --------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.out = None

    def start(self):
        try:
            self.out = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.out, stderr=subprocess.DEVNULL)
        except (OSError, FileNotFoundError):
            self.proc = None

    def stop(self) -> dict | None:
        if not self.proc:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.out.flush()
        self.out.seek(0)
        rows = [l.strip().split(", ") for l in self.out.read().splitlines() if l.strip()]
        os.unlink(self.out.name)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        loaded = [v for v in sm if v > 0.5 * (max(mx) if mx else 1)] or sm
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            for i, nm in enumerate(names):
                if len(r) > 5 + i and r[5 + i].strip().lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


# --------------------------------------------------------------- helpers
def measured_peak() -> tuple[float, str]:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        return float(json.load(open(p))["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except (OSError, KeyError, ValueError):
        return 6650.0, "fallback (B200_PROFILING.md)"


def traffic_for(kernel: str, workload: str, dtype: str = "f64"):
    """DRAM read+write bytes per launch from the committed ncu --set full
    capture of this kernel on this workload (profiles/traffic.json, written by
    tools/ncu_summary.py), if any — a cross-check of the layout bytes only."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        d = json.load(open(p))
        return d.get(workload, {}).get(kernel if dtype == "f64" else f"{kernel}:{dtype}")
    except (OSError, ValueError):
        return None


def roofline_obj(kname, layout_bytes, alg_bytes, peak, peak_src, avg_kernel_s, workload, dtype="f64") -> dict:
    """Roofline of the dominant kernel: the bytes its layout moves per launch
    (pepp_choice_t.layout_bytes: the matrix arrays as stored and streamed, x
    read once, y written once) / its average launch time (CUDA events on the
    launching stream, timed region), against the measured copy peak.
    `effective_gbs` = SURVEY §8(d)'s algorithmic bytes (nnz*12 + row_ptr +
    x + y, the metric's CSR-equivalent count) / the same time — a compressed
    layout does the same work with fewer bytes, so that figure can exceed
    the peak and is not a roofline fraction. `traffic` = ncu DRAM bytes per
    launch from the committed capture (profiles/traffic.json), a cross-check:
    `traffic_vs_layout` should be ~1 (gathers that miss L2 push it above)."""
    achieved = layout_bytes / avg_kernel_s / 1e9
    d = {"bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak, "peak_source": peak_src,
         "unit": "GB/s", "frac": round(achieved / peak, 4), "avg_launch_us": round(avg_kernel_s * 1e6, 2),
         "bytes_per_launch": int(layout_bytes), "bytes_source": "plan layout (pepp_choice_t.layout_bytes)",
         "effective_gbs": round(alg_bytes / avg_kernel_s / 1e9, 1), "algorithmic_bytes_per_launch": int(alg_bytes)}
    traffic = traffic_for(kname, workload, dtype)
    d["traffic"] = traffic
    if traffic:
        d["traffic_vs_layout"] = round(traffic / layout_bytes, 4)
        d["traffic_source"] = "ncu --set full capture committed in profiles/ (traffic.json)"
    return d


def parse_variant(s: str | None):
    import paper_conf_sc_dastgeerlk12_b200 as pepp
    if not s:
        return None
    name, _, prm = s.partition(":")
    v = {"csr_vector": pepp.V_CSR_VECTOR, "merge_path": pepp.V_MERGE_PATH, "sell": pepp.V_SELL,
         "csr_stream": pepp.V_CSR_STREAM, "panel": pepp.V_PANEL}[name]
    return pepp.Choice(v, int(prm) if prm else 0)


def cpu_baseline(A, x0: np.ndarray, iters: int, budget_s: float = 4.0) -> dict:
    """The oracle as it stands (test infrastructure), on the host cores: at
    least `iters` SpMVs, more until `budget_s` seconds of wall time."""
    import oracle
    cores = os.cpu_count()
    t0 = time.perf_counter()
    x = x0
    n = 0
    while n < iters or time.perf_counter() - t0 < budget_s:
        x = oracle.spmv(A, x, parallel=True)
        n += 1
    iters = n
    t = time.perf_counter() - t0
    gflops = 2.0 * A.nnz * iters / t / 1e9
    # single-core sequential oracle on one iteration (the paper's "serial C++" role, P@33595)
    t1 = time.perf_counter()
    oracle.spmv(A, x0, parallel=False)
    ts = time.perf_counter() - t1
    return {"value": round(gflops, 3), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
            "sample": f"{iters} full-size SpMV(s) of the bench matrix ({A.nnz} nnz) with "
                      f"oracle_spmv_rows_parallel on {cores} OpenMP threads",
            "seq_1core_gflops": round(2.0 * A.nnz / ts / 1e9, 3), "host": host_cpu()}


def host_cpu() -> dict:
    """CPU model and socket count of the host the oracle ran on."""
    model, sockets = None, set()
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                k, _, v = line.partition(":")
                k = k.strip()
                if k == "model name" and model is None:
                    model = v.strip()
                elif k == "physical id":
                    sockets.add(v.strip())
    except OSError:
        pass
    return {"model": model, "sockets": len(sockets) or None, "nproc": os.cpu_count()}


def library_baseline(A, xs, stream, iterated, flush, ours_us: float) -> dict:
    """cuSPARSE CSR SpMV (through torch.sparse_csr_tensor @ x) on the same
    matrix and x, timed with CUDA events on the same stream: context for the
    hand-written kernels, never on the product path."""
    import torch
    dev = xs.device
    it = torch.int32 if A.nnz < (1 << 31) - 1 else torch.int64
    crow = torch.from_numpy(A.row_ptr - A.row_ptr[0]).to(device=dev, dtype=it)
    col = torch.from_numpy(A.col).to(device=dev, dtype=it)
    val = torch.from_numpy(A.val).to(dev)
    M = torch.sparse_csr_tensor(crow, col, val, size=(A.nrows, A.ncols))
    del crow, col, val
    n = 10 if A.nnz > 10_000_000 else 50
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
    with torch.cuda.stream(stream):
        y = M @ xs   # warm-up (cuSPARSE buffer + analysis)
        for a, b in ev:
            if flush is not None:
                flush.zero_()
            a.record(stream)
            y = M @ xs
            b.record(stream)
    stream.synchronize()
    us = statistics.median(a.elapsed_time(b) for a, b in ev) * 1e3
    del M, y
    torch.cuda.empty_cache()
    return {"name": "cuSPARSE CSR SpMV (torch.sparse_csr_tensor @ x, torch " + torch.__version__ + ")",
            "us_per_spmv": round(us, 2), "gflops": round(2.0 * A.nnz / (us * 1e-6) / 1e9, 3),
            "speedup_ours": round(us / ours_us, 3),
            "note": "same matrix / x / stream, median of %d calls%s" % (n, "" if flush is None else ", L2 flushed")}


def value_compressed_leg(args, A, xs, bufs, stream, iters, iterated, flush, peak):
    """The same SpMVs with opts.compress_values = 1: SELL chunks whose 32 rows
    share their column offsets and whose slots hold one constant value per
    slot (constant-coefficient stencils) become ids into a pattern table in
    the kernel's parameter space, so they read only x and write y. Lossless
    and bit-identical (tests/test_gpu_parity.py::test_value_compression_lossless),
    but on the Laplacian it turns the matrix stream into a stencil: reported
    here with its own DRAM-traffic roofline, not as the headline."""
    import torch

    import paper_conf_sc_dastgeerlk12_b200 as pepp
    plan = pepp.Plan.from_csr(A, compress_values=True)
    try:
        info = plan.info()
        if info["sell_constval_frac"] <= 0:
            return {"applies": False, "note": "no constant-coefficient chunks in this matrix"}
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(iters)]
        used: dict = {}
        lbytes: dict = {}

        def step(record):
            with torch.cuda.stream(stream):
                src = xs
                for k in range(iters):
                    if not iterated:
                        src = xs
                        if flush is not None:
                            flush.zero_()
                    if record:
                        ev[k][0].record(stream)
                    u = plan.exec(src, bufs[k & 1], flags=pepp.Y_LOCAL, stream=stream)
                    if record:
                        ev[k][1].record(stream)
                        used[u.name] = used.get(u.name, 0) + 1
                        lbytes[u.name] = u.layout_bytes
                    if iterated:
                        src = bufs[k & 1]
        for _ in range(args.warmup):
            step(False)
        ms = []
        for _ in range(max(1, min(args.steps, 5))):
            step(True)
            stream.synchronize()
            ms.extend(a.elapsed_time(b) for a, b in ev)
        avg_s = statistics.mean(ms) / 1e3
        chosen = max(used, key=used.get)
        kname = chosen + ("+constval" if chosen.startswith("sell") else "")
        lb = lbytes[chosen]
        traffic = traffic_for(kname, args.workload, args.dtype)
        d = {"applies": True, "kernel": kname, "constval_frac": info["sell_constval_frac"],
             "avg_launch_us": round(avg_s * 1e6, 2), "gflops": round(2.0 * A.nnz / avg_s / 1e9, 3),
             "layout_bytes": lb, "achieved_gbs": round(lb / avg_s / 1e9, 1),
             "frac": round(lb / avg_s / 1e9 / peak, 4), "traffic": traffic, "choices": used,
             "note": "opts.compress_values = 1: constant stencil chunks read only x and write y; lossless; "
                     "frac = layout bytes (x read once, y written, lists) / launch time / measured peak"}
        if traffic:
            d["traffic_vs_layout"] = round(traffic / lb, 4)
        return d
    finally:
        plan.close()


LEG_WORKLOADS = ("lap64", "uniform1m", "zipf4m")   # BASELINE configs 1, 2, 3


def config_leg(name: str, args, dev, stream, peak: float, with_cpu: bool) -> dict:
    """One of BASELINE's single-SpMV configs measured beside the headline (rank
    0, N = 1): plan time (matrix upload + layouts), the automatic choice's
    median time per SpMV after calibration (kernel events, L2 flushed between
    calls), its layout bytes / time against the measured peak, every
    candidate forced (selector ratio = chosen / best), a cold single call with
    the matrix upload (plan + pepp_spmv_exec_host: x in, y out), and the CPU
    oracle's time for one SpMV (break-even call count = plan / (cpu - gpu))."""
    import torch

    import paper_conf_sc_dastgeerlk12_b200 as pepp
    R = len(global_rowptr(name)) - 1
    A = make_block(name, 0, R)
    x0 = x0_vector(name, A.ncols)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    plan = pepp.Plan.from_csr(A)
    torch.cuda.synchronize()
    plan_ms = (time.perf_counter() - t0) * 1e3
    try:
        yh = torch.empty(A.nrows, dtype=torch.float64).pin_memory().numpy()
        xh = torch.from_numpy(x0).pin_memory().numpy()
        t1 = time.perf_counter()
        plan.exec_host(xh, yh, iterations=1, stream=stream)      # first call: cold, with its copies
        cold_call_ms = (time.perf_counter() - t1) * 1e3
        xs = torch.from_numpy(x0).to(dev)
        y = torch.empty(A.nrows, dtype=torch.float64, device=dev)
        small = A.nnz < 100_000
        flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
        ncal = 200 if small else 40
        with torch.cuda.stream(stream):
            for _ in range(ncal):   # calibration (history-based selection settles)
                plan.exec(xs, y, stream=stream)
        stream.synchronize()
        n = 200 if small else 30
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        used: dict = {}
        lb: dict = {}
        with torch.cuda.stream(stream):
            for a, b in ev:
                flush.zero_()
                a.record(stream)
                u = plan.exec(xs, y, stream=stream)
                b.record(stream)
                used[u.name] = used.get(u.name, 0) + 1
                lb[u.name] = u.layout_bytes
        stream.synchronize()
        us = statistics.median(a.elapsed_time(b) for a, b in ev) * 1e3
        chosen = max(used, key=used.get)
        per = {}
        for c in plan.candidates():
            f = pepp.Choice(c.variant, c.param)
            m = 40 if small else 10
            pairs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(m)]
            with torch.cuda.stream(stream):
                for a, b in pairs:
                    flush.zero_()
                    a.record(stream)
                    plan.exec(xs, y, stream=stream, force=f)
                    b.record(stream)
            stream.synchronize()
            per[f.name] = statistics.median(a.elapsed_time(b) for a, b in pairs[2:]) * 1e3
        best = min(per, key=per.get)
        graph_us = None
        if small:   # launch-bound: the same call replayed from a CUDA graph
            g = plan.graph(xs, y, iterations=1000, mode=0, stream=stream)
            with torch.cuda.stream(stream):
                g.launch(stream)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                for _ in range(5):
                    g.launch(stream)
                e1.record(stream)
            e1.synchronize()
            graph_us = round(e0.elapsed_time(e1) * 1e3 / 5000, 3)
            g.close()
        alg = A.nnz * 12 + (A.nrows + 1) * 4 + A.ncols * 8 + A.nrows * 8
        d = {"desc": WORKLOADS[name]["desc"], "rows": A.nrows, "nnz": A.nnz, "chosen": chosen,
             "us_per_spmv": round(us, 2), "gflops": round(2.0 * A.nnz / (us * 1e-6) / 1e9, 2),
             "layout_bytes": lb[chosen], "achieved_gbs": round(lb[chosen] / (us * 1e-6) / 1e9, 1),
             "frac": round(lb[chosen] / (us * 1e-6) / 1e9 / peak, 4),
             "effective_gbs": round(alg / (us * 1e-6) / 1e9, 1),
             "selector": {"best": best, "best_us": round(per[best], 2), "ratio": round(per.get(chosen, us) / per[best], 4),
                          "candidates_us": {k: round(v, 2) for k, v in per.items()}},
             "plan_ms": round(plan_ms, 1), "cold_call_incl_copies_ms": round(cold_call_ms, 3),
             "e2e_single_call_incl_upload_ms": round(plan_ms + cold_call_ms, 1),
             "graph_us_per_call": graph_us}
        if small:
            d["note"] = "launch-latency bound (20 K nnz): frac not a roofline claim; see graph_us_per_call"
        if name in ("uniform1m", "zipf4m", "skew"):
            # random columns: one x gather (a 32-B sector for 8 B) per stored
            # entry; the ceiling is the measured random-gather rate from an
            # L2-resident x, not HBM bandwidth
            gps = A.nnz / (us * 1e-6)
            d["gather_bound"] = {"gathers_per_spmv": int(A.nnz), "achieved_g_per_s": round(gps / 1e9, 1),
                                 "ceiling_g_per_s": GATHER_CEILING_G, "frac": round(gps / 1e9 / GATHER_CEILING_G, 4),
                                 "ceiling_source": "tools/experiments/gather_probe.cu: random 8-B gathers from an "
                                                   "L2-resident x on this B200 pool, any load path (DESIGN §6)"}
        if with_cpu:
            import oracle
            t2 = time.perf_counter()
            reps = 0
            while reps < 3 or time.perf_counter() - t2 < 0.5:
                oracle.spmv(A, x0, parallel=True)
                reps += 1
            cpu_ms = (time.perf_counter() - t2) * 1e3 / reps
            d["cpu_oracle_ms"] = round(cpu_ms, 3)
            gap = cpu_ms - us * 1e-3
            d["break_even_calls"] = round(plan_ms / gap, 1) if gap > 0 else None
        return d
    finally:
        plan.close()
        torch.cuda.empty_cache()


GATHER_CEILING_G = 255.0   # G random 8-B gathers / s from L2 (measured)

# --------------------------------------------------------------- arms
METRIC = "SpMV GFLOP/s (aggregate over ranks); achieved HBM GB/s in 'hbm'"


def config_of(args, R: int, Z: int) -> dict:
    """The workload description both arms print (same dict, same keys)."""
    wl = WORKLOADS[args.workload]
    iters = args.iters or wl["iters"]
    alg = Z * 12 + (R + 1) * 4 + R * 16
    l2 = (f"inputs larger than L2 ({alg / 1e9:.1f} GB/SpMV)" if wl["iterated"]
          else "L2 flushed (512 MB memset) between SpMVs; kernel events only" if alg < 4 * (1 << 30)
          else f"inputs larger than L2 ({alg / 1e9:.1f} GB/SpMV)")
    return {"workload": args.workload, "desc": wl["desc"], "spmv_per_step": iters, "rows": R, "nnz": Z, "l2": l2}


def run_reference(args, rank: int, world: int) -> None:
    """--impl reference: the CPU oracle (no code was published with the paper)."""
    if rank != 0:
        return
    import oracle
    wl = WORKLOADS[args.workload]
    A = make_block(args.workload, 0, len(global_rowptr(args.workload)) - 1)
    x = x0_vector(args.workload, A.ncols)
    for _ in range(args.warmup):
        oracle.spmv(A, x, parallel=True)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.spmv(A, x, parallel=True)
    t = time.perf_counter() - t0
    flops = 2.0 * A.nnz * args.steps
    val = flops / t / 1e9
    cores = os.cpu_count()
    sample = (f"each step = 1 of the {wl['iters']} SpMVs of a {args.workload} step, full matrix "
              f"({A.nnz} nnz), oracle_spmv_rows_parallel on {cores} threads")
    line = {"impl": "reference", "metric": METRIC, "value": round(val, 3), "unit": "GFLOP/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1000 * t / args.steps, 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": config_of(args, A.nrows, A.nnz),
            "cpu_baseline": {"value": round(val, 3), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                             "sample": sample, "host": host_cpu()},
            "e2e": {"value": round(val, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_ours(args, rank: int, world: int, local_rank: int) -> None:
    import torch
    import torch.distributed as dist

    import paper_conf_sc_dastgeerlk12_b200 as pepp

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    wl = WORKLOADS[args.workload]
    iters = args.iters or wl["iters"]
    iterated = wl["iterated"]

    # ---- partition (a2) + this rank's block ----
    rp_global = global_rowptr(args.workload)
    R = len(rp_global) - 1
    Z = int(rp_global[-1])
    bounds = pepp.partition_rows(rp_global, world)
    r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
    del rp_global
    A = make_block(args.workload, r0, r1)
    x0 = x0_vector(args.workload, A.ncols)
    f32 = args.dtype == "f32"
    if f32:   # the fp32 instance (paper's `float` signature): same matrix, values rounded to float
        import gen
        A = gen.CSR(A.nrows, A.ncols, A.row_ptr, A.col, A.val.astype(np.float32), A.r0, A.global_nrows, A.name)
        x0 = x0.astype(np.float32)
    tdt = torch.float32 if f32 else torch.float64
    esz = 4 if f32 else 8

    uid = None
    if world > 1:
        obj = [pepp.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    force = parse_variant(args.variant)
    # --variant pins the choice everywhere (timed steps and the e2e leg): the
    # plan is built with that variant only
    # plan = matrix upload (host -> device) + validation + every variant's
    # layout (a1-a3), timed: the cost a caller pays once before any call
    torch.cuda.synchronize()
    t_plan = time.perf_counter()
    plan = pepp.Plan.from_csr(A, nranks=world, rank=rank, row_bounds=bounds if world > 1 else None,
                              nccl_unique_id=uid, prune=not args.no_prune,
                              variant_mask=(1 << force.variant) if force is not None else 0,
                              compress_values=args.value_compression)
    torch.cuda.synchronize()
    plan_ms = (time.perf_counter() - t_plan) * 1e3
    info = plan.info()
    flags = pepp.Y_NEXT_INPUT if iterated else pepp.Y_LOCAL
    # N > 1, iterated: the exchange happens inside each call, as the plan's
    # distribution choice (P', exchange — opts.dist_select) or its overlapped halo
    overlapped = bool(world > 1 and iterated and force is None)

    stream = torch.cuda.Stream(device=dev)
    xs = torch.from_numpy(x0).to(dev)
    p2p = overlapped and bool(info["overlap"]) and not args.no_p2p
    p2p_note = None
    bufs = None
    if p2p:
        # symmetric buffers: the boundary kernel pushes the halo straight into
        # the neighbours' copies over peer memory (PEPP_X_P2P), no NCCL per
        # iteration. The library's registration is agreed on by every rank:
        # if any rank cannot map its peers (no CUDA IPC / peer access) or
        # cannot take part, all ranks get the same error and the plan keeps
        # the NCCL halo — fall back to it here.
        try:
            bufs = plan.p2p_buffers(2)
        except pepp.PeppError as e:
            p2p, p2p_note = False, f"p2p unavailable, NCCL halo used: {e}"[:300]
    if bufs is None:
        bufs = [torch.empty(R, dtype=tdt, device=dev) for _ in range(2)]
    final_info = plan.info()   # after the P2P registration (its timing may change the distribution choice)
    flush = None if iterated or Z * 12 > 4 * (1 << 30) else torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    ev_pool = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(iters)]
    launches = {"n": 0}
    used_count: dict = {}
    used_bytes: dict = {}

    def one_step(record: bool):
        """`iters` SpMVs through the C-ABI. Iterated: x0 -> b0 -> b1 -> b0 ...
        (x0 stays resident and is only read, so every step restarts from it)."""
        kernel_ms = []
        with torch.cuda.stream(stream):
            src = xs
            for k in range(iters):
                dst = bufs[k & 1]
                if not iterated:
                    src = xs
                    if flush is not None:
                        flush.zero_()
                a, b = ev_pool[k]
                if record:
                    a.record(stream)
                if overlapped:
                    # halo exchange overlapped with the interior rows inside the call:
                    # the events bracket kernels + exchange
                    u = plan.exec(src, dst, flags=flags, stream=stream)
                else:
                    # kernel (events bracket it alone), then the exchange step
                    u = plan.exec(src, dst, flags=pepp.Y_LOCAL, stream=stream, force=force)
                if record:
                    b.record(stream)
                    used_count[u.name] = used_count.get(u.name, 0) + 1
                    used_bytes[u.name] = u.layout_bytes
                    launches["n"] += u.launches   # the library's own count of its kernels in this call
                if not overlapped and flags != pepp.Y_LOCAL and world > 1:
                    plan.exchange(dst, flags, stream=stream)
                if iterated:
                    src = dst
        return kernel_ms

    def barrier():
        if world > 1:
            dist.barrier()

    def allmax(v: float) -> float:
        """max over ranks (device tensor for NCCL, host tensor for gloo)"""
        if world == 1:
            return v
        on_dev = dist.get_backend() == "nccl"
        t = torch.tensor([v], dtype=torch.float64, device=dev if on_dev else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # one cold call (fresh plan, first launch of the process's kernels on this
    # matrix) — reported for launch-bound workloads
    cold_us = None
    if not iterated and A.nnz < 10_000_000:
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        with torch.cuda.stream(stream):
            c0.record(stream)
            plan.exec(xs, bufs[0], flags=flags, stream=stream)
            c1.record(stream)
        c1.synchronize()
        cold_us = round(c0.elapsed_time(c1) * 1e3, 2)
    for _ in range(args.warmup):
        one_step(False)
    torch.cuda.synchronize()
    barrier()

    # ---- timed region ----
    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    barrier()
    torch.cuda.synchronize()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    kern_ms = []
    t_start.record(stream)
    for _ in range(args.steps):
        one_step(True)
        # harvest this step's per-launch kernel times (the events are reused next step)
        torch.cuda.current_stream(dev).wait_stream(stream)
        stream.synchronize()
        kern_ms.extend(a.elapsed_time(b) for a, b in ev_pool)
    t_end.record(stream)
    torch.cuda.synchronize()
    barrier()
    clk = clocks.stop()
    total_ms = allmax(t_start.elapsed_time(t_end))

    nspmv = iters * args.steps
    alg_bytes_global = Z * (4 + esz) + (R + 1) * 4 + A.ncols * esz + R * esz
    if iterated:
        secs = total_ms / 1e3
    else:
        # single-SpMV workloads: L2 flushed between calls; time = sum of kernel events
        secs = allmax(sum(kern_ms) / 1e3)
    gflops = 2.0 * Z * nspmv / secs / 1e9
    gbs = alg_bytes_global * nspmv / secs / 1e9
    peak, peak_src = measured_peak()

    # roofline of the dominant kernel on this rank (rank 0 reports)
    avg_kernel_s = statistics.mean(kern_ms) / 1e3
    local_alg = A.nnz * (4 + esz) + (A.nrows + 1) * 4 + (A.nrows + info["halo_recv"]) * esz + A.nrows * esz
    if world == 1:
        local_alg = alg_bytes_global
    chosen = max(used_count, key=used_count.get) if used_count else "?"
    layout_bytes = used_bytes.get(chosen, local_alg)
    if overlapped:   # the call's `used` is the interior sub-plan's: use the whole block's layout of that variant
        for c in plan.candidates():
            if c.name == chosen:
                layout_bytes = c.layout_bytes

    # ---- the value-compressed layout (opts.compress_values), reported beside the headline ----
    vc = None
    if world == 1 and not args.value_compression and force is None and not args.no_vc_leg:
        vc = value_compressed_leg(args, A, xs, bufs, stream, iters, iterated, flush, peak)

    # ---- cuSPARSE on the same matrix (context, not the product path) ----
    lib_base = None
    if world == 1 and not args.no_library:
        try:
            lib_base = library_baseline(A, xs, stream, iterated, flush, avg_kernel_s * 1e6)
        except Exception as e:   # context only: never fail the bench line over it
            lib_base = {"unavailable": repr(e)[:200]}

    # ---- selector quality: every candidate timed after the timed region (same run) ----
    sel = None
    if not args.no_sweep:
        per = {}
        for c in plan.candidates():
            f = pepp.Choice(c.variant, c.param)
            # issued back to back like the timed region (events around each
            # call, no host sync in between): small matrices get more calls,
            # their per-call times are a few microseconds
            ncall = min(iters, 10 if A.nnz > 10_000_000 else 100) + 2
            pairs = []
            with torch.cuda.stream(stream):
                src = xs
                for k in range(ncall):
                    if flush is not None:
                        flush.zero_()
                    a, b = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                    a.record(stream)
                    plan.exec(src, bufs[k & 1], flags=flags, stream=stream, force=f)
                    b.record(stream)
                    pairs.append((a, b))
                    if iterated:
                        src = bufs[k & 1]
            stream.synchronize()
            ts = [a.elapsed_time(b) for a, b in pairs[2:]]
            per[f.name] = statistics.median(ts) * 1e3
        best = min(per, key=per.get)
        sel = {"chosen": chosen, "chosen_us": round(per.get(chosen, float("nan")), 2), "best": best,
               "best_us": round(per[best], 2), "ratio": round(per.get(chosen, float("nan")) / per[best], 4),
               "candidates_us": {k: round(v, 2) for k, v in per.items()}}

    # ---- launch-bound workloads: the same calls replayed from a CUDA graph ----
    graph_info = None
    if not iterated and A.nnz < 10_000_000:
        ncalls = 1000
        g = plan.graph(xs, bufs[0], iterations=ncalls, mode=0, stream=stream)
        with torch.cuda.stream(stream):
            g.launch(stream)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            reps = 5
            for _ in range(reps):
                g.launch(stream)
            e1.record(stream)
        e1.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / (reps * ncalls)
        graph_info = {"calls": ncalls, "us_per_call": round(us, 3), "cold_first_call_us": cold_us,
                      "gflops": round(2.0 * Z / (us * 1e-6) / 1e9, 3),
                      "note": "back-to-back calls replayed from one CUDA graph (pepp_spmv_graph_*); L2-warm"}
        g.close()

    # ---- e2e: host buffers through the C-ABI (pepp_spmv_exec_host) ----
    # every step copies its own x in from pinned host memory and its y out;
    # pepp_spmv_exec_host_batch overlaps step k+1's input copy and step
    # k-1's output copy with step k's SpMVs (two pinned x / y buffers alternate)
    xh = [torch.from_numpy(x0).pin_memory().numpy() for _ in range(2)]
    yh = [torch.empty(R, dtype=tdt).pin_memory().numpy() for _ in range(2)]
    e2e_iters = iters if iterated else 1
    e2e_flags = flags
    e2e_steps = max(2, args.steps)
    xs_list = [xh[k & 1] for k in range(e2e_steps)]
    ys_list = [yh[k & 1] for k in range(e2e_steps)]
    plan.exec_host_batch(xs_list[:2], ys_list[:2], iterations=e2e_iters, flags=e2e_flags, stream=stream)   # warm
    barrier()
    te = time.perf_counter()
    plan.exec_host_batch(xs_list, ys_list, iterations=e2e_iters, flags=e2e_flags, stream=stream)
    te = allmax(time.perf_counter() - te)
    e2e_val = 2.0 * Z * e2e_iters * e2e_steps / te / 1e9

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu and not f32:
        cpu = cpu_baseline(A, x0, 2 if A.nnz > 10_000_000 else 200)

    # transfer- and plan-inclusive view (the paper's Fig. 5 setting, P@35591-35720)
    step_s = te / e2e_steps
    with_plan = {"plan_ms": round(plan_ms, 1),
                 "first_step_incl_plan_gflops": round(2.0 * Z * e2e_iters / (plan_ms / 1e3 + step_s) / 1e9, 3),
                 "note": "one e2e step (host x in, iterations, host y out) plus the plan that uploads the matrix"}
    if cpu:
        t_cpu = 2.0 * Z / (cpu["value"] * 1e9)
        t_gpu = secs / nspmv
        with_plan["break_even_spmvs_vs_cpu_oracle"] = round(plan_ms / 1e3 / (t_cpu - t_gpu), 1) if t_cpu > t_gpu else None

    # BASELINE configs 1-3 beside the headline (rank 0, N = 1, default workload)
    legs = None
    if rank == 0 and world == 1 and args.workload == "lap8192" and not args.no_legs and not f32 and force is None:
        legs = {}
        for name in LEG_WORKLOADS:
            try:
                legs[name] = config_leg(name, args, dev, stream, peak, with_cpu=not args.no_cpu)
            except Exception as e:   # reported, never fatal for the headline
                legs[name] = {"error": repr(e)[:300]}

    if rank == 0:
        kname = chosen
        if kname.startswith("sell") and info["sell_constval_frac"] > 0:
            kname += "+constval"   # value-compressed layout: its own ncu traffic entry
        line = {
            "metric": METRIC,
            "value": round(gflops, 3), "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": config_of(args, R, Z),
            "run": {"exchange": ("p2p (fused boundary kernel, peer-memory stores)"
                                 if final_info["dist_exchange"] == pepp.X_P2P or (p2p and not final_info["dist_candidates"])
                                 else pepp._capi.EXCHANGE_NAMES.get(final_info["dist_exchange"] if final_info["dist_candidates"]
                                                                    else info["exchange"], "?")),
                    "nparts": final_info["dist_nparts"] if final_info["dist_candidates"] else world,
                    "distribution": ([{"nparts": a, "exchange": pepp._capi.EXCHANGE_NAMES.get(b, "?"),
                                       "agreed_us": round(c, 2)} for a, b, c in plan.dist_stats()]
                                     if final_info["dist_candidates"] else None),
                    "dist_probe_ms": round(final_info["dist_probe_ms"], 1),
                    "p2p_fallback": p2p_note,
                    "variant": args.variant or "auto (history-based per call)",
                    "plan_ms": round(plan_ms, 1),
                    "plan_note": "pepp_spmv_plan wall time on rank 0: host -> device copy of the matrix, "
                                 "validation, context extraction and every variant's layout (a1-a3); paid once"},
            "hbm": {"achieved_gbs": round(gbs, 1), "frac_of_measured": round(gbs / (world * peak), 4),
                    "frac_of_8tbs": round(gbs / (world * 8000.0), 4), "algorithmic_bytes_per_spmv": alg_bytes_global,
                    "note": "BASELINE's metric count (SURVEY 8(d): nnz*12 B + row_ptr + x + y per SpMV over the step "
                            "time); the chosen layout moves fewer bytes for the same work, so these fractions can "
                            "exceed 1 — the physical fraction is roofline.frac (layout bytes / launch time)"},
            "roofline": dict(roofline_obj(kname, layout_bytes, local_alg, peak, peak_src, avg_kernel_s, args.workload, args.dtype),
                             **({"launch_includes": "the whole call: its kernels and its exchange, as the plan's "
                                                    "distribution choice runs them (run.nparts / run.exchange)"}
                                if overlapped else {})),
            "e2e": {"value": round(e2e_val, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": A.ncols * esz,
                    "d2h_bytes_per_step": A.nrows * esz, "spmv_per_step": e2e_iters,
                    "steps": e2e_steps,
                    "api": "pepp_spmv_exec_host_batch (per step: pinned host x -> device, iterations, device -> "
                           "pinned host y; step k+1's input copy and step k-1's output copy overlap step k)",
                    "with_plan": with_plan},
            "configs": legs,
            "gpu_launches": launches["n"],
            "graph": graph_info,
            "selector": sel,
            "value_compressed": vc,
            "library_baseline": lib_base,
            "clocks": clk,
            "cpu_baseline": cpu,
            "plan": {k: info[k] for k in ("mean_row", "cv_row", "max_row", "sell_sigma", "sell_fill",
                                          "sell_stencil_frac", "sell_constval_frac", "sell_col16_frac",
                                          "device_bytes", "halo_recv", "halo_send", "overlap",
                                          "overlap_head", "overlap_tail")},
            "choices": used_count,
        }
        print(json.dumps(line), flush=True)
    plan.close()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=sorted(WORKLOADS), default="lap8192")
    ap.add_argument("--iters", type=int, default=0)
    ap.add_argument("--variant", default=None)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-sweep", action="store_true")
    ap.add_argument("--no-prune", action="store_true", help="every variant is a candidate (no static narrowing)")
    ap.add_argument("--value-compression", action="store_true",
                    help="headline plan with opts.compress_values = 1 (constant-coefficient stencil chunks "
                         "stored as pattern-table ids, values not streamed); default: every stored value is "
                         "streamed and the compressed plan is reported separately under 'value_compressed'")
    ap.add_argument("--no-value-compression", action="store_true", help=argparse.SUPPRESS)   # the default now
    ap.add_argument("--no-vc-leg", action="store_true", help="skip the value-compressed leg")
    ap.add_argument("--no-library", action="store_true", help="skip the cuSPARSE context measurement")
    ap.add_argument("--no-legs", action="store_true", help="skip the BASELINE config 1-3 legs of the default line")
    ap.add_argument("--no-p2p", action="store_true",
                    help="N > 1: NCCL halo per iteration instead of the fused peer-memory push (PEPP_X_P2P)")
    ap.add_argument("--dtype", choices=["f64", "f32"], default="f64",
                    help="f64 = BASELINE's precision (default); f32 = the paper's float instance")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # `python bench.py --gpus N` on its own: one process per GPU, launched
        # the way the driver launches N > 1 (torch.distributed.run, 127.0.0.1)
        import socket
        sk = socket.socket()
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
        sk.close()
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(args.gpus),
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *sys.argv[1:]]
        sys.exit(subprocess.call(cmd))

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (one process per GPU)")
    if world > 1:
        # NCCL's communicator init lines (rank, nranks, transport) in the log:
        # evidence of the N-rank communicators the library and torch build
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    # Test-only knobs (tests/test_gpu_bench_multirank.py): run every rank on one
    # device with gloo for torch.distributed (the library then needs
    # PEPP_NCCL_LIB pointing at the NCCL stand-in). Never set by the driver.
    if os.environ.get("PEPP_BENCH_ONE_DEVICE"):
        local_rank = 0
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        backend = os.environ.get("PEPP_BENCH_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(backend)
    try:
        if args.impl == "reference":
            run_reference(args, rank, world)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
