"""Config-5-style sweep of the distribution choice (row a4: P' and exchange)
with two ranks on ONE GPU: the library's NCCL entry points are served by the
test stand-in (tests/support/fake_nccl.c — host-staged, so the absolute
exchange times are those of the stand-in, not NVLink), CUDA IPC for the
fused push. Per matrix: the plan's agreed choice (plan-time timing,
max-over-ranks means) against an exhaustive timing of every candidate
forced afterwards (mean of iterated NEXT_INPUT calls, device events around
the whole call, max over ranks): ratio = chosen / best.

  python tools/r2/dist_sweep.py [--out profiles/r2_dist_sweep.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))


def worker(rank, world, lib, uid, kind, n, q):
    try:
        work(rank, world, lib, uid, kind, n, q)
    except Exception as e:
        import traceback
        q.put((rank, {"error": repr(e) + traceback.format_exc()}))


def work(rank, world, lib, uid, kind, n, q):
    os.environ["PEPP_NCCL_LIB"] = lib
    os.environ["PEPP_FAKE_NCCL_BOX_MB"] = "320"   # P' = 1 ships a whole row block in one message at plan time
    sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import gen
    import paper_conf_sc_dastgeerlk12_b200 as pepp
    torch.cuda.set_device(0)
    A = gen.banded(n, 4, seed=100) if kind == "banded" else gen.uniform(n, n, 16, seed=100)
    bounds = pepp.partition_rows(A.row_ptr, world)
    blk = gen.row_block(A, int(bounds[rank]), int(bounds[rank + 1]))
    with pepp.Plan.from_csr(blk, nranks=world, rank=rank, row_bounds=bounds, nccl_unique_id=uid) as plan:
        info = plan.info()
        bufs = plan.p2p_buffers(2) if info["overlap"] else None
        if bufs is None:
            bufs = [torch.zeros(n, dtype=torch.float64, device="cuda") for _ in range(2)]
        info = plan.info()
        stats = plan.dist_stats()
        res = {"chosen": (info["dist_nparts"], info["dist_exchange"]), "agreed": stats, "forced": {}}
        for parts, ex, _ in stats:
            f = pepp.Choice(pepp._capi.V_AUTO, 0, exchange=ex, nparts=parts)
            ts = []
            for k in range(12):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                plan.exec(bufs[k & 1], bufs[(k + 1) & 1], flags=pepp.Y_NEXT_INPUT, force=f)
                b.record()
                b.synchronize()
                ts.append(a.elapsed_time(b) * 1e3)
            res["forced"][f"{parts}:{ex}"] = statistics.mean(ts[2:])
        q.put((rank, res))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "dist_sweep.jsonl"))
    ap.add_argument("--timeout", type=float, default=300)
    ap.add_argument("--sizes", default="1e4,1e5,1e6")
    ap.add_argument("--kinds", default="banded,uniform")
    a = ap.parse_args()
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    from test_gpu_partitioned import _build_fake
    import torch.multiprocessing as mp
    lib = _build_fake()
    names = {1: "allgather", 2: "halo", 3: "p2p"}
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    fo = open(a.out, "w")
    for kind in a.kinds.split(","):
        for n in [int(float(v)) for v in a.sizes.split(",")]:
            uid = (f"/tmp/pepp_fake_nccl_{os.getpid()}_{kind}_{n}".encode() + b"\0" * 128)[:128]
            ctx = mp.get_context("spawn")
            q = ctx.Queue()
            ps = [ctx.Process(target=worker, args=(r, 2, lib, uid, kind, n, q)) for r in range(2)]
            for p in ps:
                p.start()
            out = {}
            try:
                for _ in range(2):
                    r, res = q.get(timeout=a.timeout)
                    out[r] = res
            except Exception as e:   # a stuck rank: report and go on
                out.setdefault(0, {"error": "timeout " + repr(e)})
            finally:
                for p in ps:
                    p.join(30)
                    if p.is_alive():
                        p.kill()
            if len(out) < 2 or any("error" in out[r] for r in out):
                print(json.dumps({"kind": kind, "rows": n, "error": {r: out[r].get("error", "")[-1500:] for r in out}}), flush=True)
                continue
            forced = {k: max(out[r]["forced"][k] for r in range(2)) for k in out[0]["forced"]}
            best = min(forced, key=forced.get)
            ch = "%d:%d" % tuple(out[0]["chosen"])
            line = {"kind": kind, "rows": n, "ranks": 2, "chosen": ch, "chosen_us": round(forced[ch], 1),
                    "best": best, "best_us": round(forced[best], 1), "ratio": round(forced[ch] / forced[best], 3),
                    "ranks_agree": out[0]["chosen"] == out[1]["chosen"],
                    "agreed_us": {f"{p}:{names.get(e, e)}": round(t, 1) for p, e, t in out[0]["agreed"]},
                    "forced_us": {k: round(v, 1) for k, v in forced.items()},
                    "transport": "fake NCCL (host-staged stand-in) + CUDA IPC on one B200"}
            print(json.dumps(line), flush=True)
            fo.write(json.dumps(line) + "\n")
            fo.flush()
    fo.close()


if __name__ == "__main__":
    main()
