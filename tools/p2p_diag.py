"""Diagnostic: the fused peer-memory halo with two processes on one GPU,
stage-by-stage timestamps per rank, hard time limits, children killed on exit."""
import faulthandler
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def log(rank, msg, t0=[time.time()]):
    line = f"[r{rank} {time.time() - t0[0]:7.2f}s] {msg}"
    print(line, flush=True)
    with open(os.path.join(ROOT, "gpurun_out", f"p2p_diag_r{rank}.log"), "a") as f:
        f.write(line + "\n")


def worker(rank, lib, uid, K, q):
    faulthandler.dump_traceback_later(90, exit=True)
    os.environ["PEPP_NCCL_LIB"] = lib
    os.environ.setdefault("PEPP_P2P_TIMEOUT_MS", "3000")
    try:
        import numpy as np
        import torch

        import gen
        import oracle
        import paper_conf_sc_dastgeerlk12_b200 as pepp
        torch.cuda.set_device(0)
        log(rank, "imported")
        A = gen.laplacian2d(96)
        bounds = pepp.partition_rows(A.row_ptr, 2)
        blk = gen.row_block(A, int(bounds[rank]), int(bounds[rank + 1]))
        x0 = gen.vector(3, gen.INT8, A.nrows)
        plan = pepp.Plan.from_csr(blk, nranks=2, rank=rank, row_bounds=bounds, nccl_unique_id=uid, exchange=pepp.X_HALO)
        log(rank, f"planned overlap={plan.info()['overlap']}")
        bufs = plan.p2p_buffers(2)
        log(rank, "p2p_buffers ok")
        bufs[0].copy_(torch.from_numpy(x0).cuda())
        bufs[1].fill_(float("nan"))
        torch.cuda.synchronize()
        log(rank, "filled")
        src, dst = bufs[0], bufs[1]
        ref = x0
        ok = True
        for k in range(K):
            u = plan.exec(src, dst, flags=pepp.Y_NEXT_INPUT)
            log(rank, f"exec {k} enqueued exchange={u.exchange}")
            torch.cuda.synchronize()
            log(rank, f"exec {k} done")
            ref = oracle.spmv(A, ref)
            y = dst.cpu().numpy()
            r0, r1 = int(bounds[rank]), int(bounds[rank + 1])
            ok &= bool(np.array_equal(y[r0:r1], ref[r0:r1]))
            src, dst = dst, src
        log(rank, f"result ok={ok}")
        plan.close()
        log(rank, "closed")
        q.put((rank, ok))
    except Exception as e:
        import traceback
        log(rank, "ERROR " + repr(e) + traceback.format_exc())
        q.put((rank, repr(e)))


def main():
    import torch.multiprocessing as mp
    from test_gpu_partitioned import _build_fake
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    lib = _build_fake()
    uid = (f"/tmp/pepp_fake_nccl_{os.getpid()}_diag".encode() + b"\0" * 128)[:128]
    K = int(sys.argv[1]) if len(sys.argv) > 1 else 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=worker, args=(r, lib, uid, K, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = {}
    t0 = time.time()
    try:
        while len(res) < 2 and time.time() - t0 < 120:
            try:
                r, v = q.get(timeout=5)
                res[r] = v
            except Exception:
                pass
    finally:
        for p in ps:
            if p.is_alive():
                p.kill()
            p.join(5)
    print("RESULT", res, flush=True)


if __name__ == "__main__":
    main()
