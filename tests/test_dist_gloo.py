"""Partitioned (multi-rank) path, CPU only: world_size 2 over gloo.

The library's host logic decides the partition (pepp_partition_rows) and
each rank's ghost columns (pepp_halo_ghosts); the ranks then run the same
exchange protocol the plan runs over NCCL (setup_halo / exchange_halo in
plan.cu: counts, then index lists, then per-peer values every iteration),
here with gloo, and compute their row block with the CPU oracle. Entries a
rank neither owns nor receives are poisoned with NaN, so an incomplete
ghost list cannot pass. Result: iterated SpMV over the concatenated row
blocks (§IV-F, P@27875) equals the unpartitioned oracle bit for bit on
integer-valued inputs (and for the allgather exchange too).
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _matrix(name):
    import gen
    if name == "lap":
        return gen.laplacian2d(24)
    if name == "zipf":
        return gen.zipf(3000, 3000, seed=47, kmax=60, val_mode=gen.INT4)
    if name == "banded":
        return gen.banded(2000, 4, seed=100, val_mode=gen.INT4)
    raise ValueError(name)


def _worker(rank, world, port, name, exchange, K, outq):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import gen
        import oracle
        import paper_conf_sc_dastgeerlk12_b200 as pepp
        dist.init_process_group("gloo", rank=rank, world_size=world)
        A = _matrix(name)
        n = A.nrows
        x0 = gen.vector(3, gen.INT8, n) if name != "lap" else gen.vector(3, gen.INT8, n)
        bounds = pepp.partition_rows(A.row_ptr, world)
        lo, hi = int(bounds[rank]), int(bounds[rank + 1])
        blk = gen.row_block(A, lo, hi)
        counts, ghosts = pepp.halo_ghosts(blk.col, world, rank, bounds)
        # --- setup: tell each peer which of its entries I need (counts, then lists)
        send_lists = {}
        recv_lists = {q: ghosts[(ghosts >= bounds[q]) & (ghosts < bounds[q + 1])] for q in range(world) if q != rank}
        for q in range(world):
            if q == rank:
                continue
            c_out = torch.tensor([len(recv_lists[q])], dtype=torch.int64)
            c_in = torch.zeros(1, dtype=torch.int64)
            if rank < q:
                dist.send(c_out, q); dist.recv(c_in, q)
            else:
                dist.recv(c_in, q); dist.send(c_out, q)
            lst_in = torch.zeros(int(c_in.item()), dtype=torch.int32)
            lst_out = torch.from_numpy(recv_lists[q].astype(np.int32))
            if rank < q:
                if lst_out.numel(): dist.send(lst_out, q)
                if lst_in.numel(): dist.recv(lst_in, q)
            else:
                if lst_in.numel(): dist.recv(lst_in, q)
                if lst_out.numel(): dist.send(lst_out, q)
            send_lists[q] = lst_in.numpy()
            # what a peer asks for must be mine
            assert np.all((send_lists[q] >= lo) & (send_lists[q] < hi))
        # --- iterate: x holds own rows + ghosts, NaN elsewhere
        x = np.full(n, np.nan)
        x[:] = x0   # iteration 0: everyone has x0
        for _ in range(K):
            y = np.full(n, np.nan)
            y[lo:hi] = oracle.spmv(blk, x)
            if exchange == "halo":
                for q in range(world):
                    if q == rank:
                        continue
                    out = torch.from_numpy(y[send_lists[q]].copy())
                    inc = torch.zeros(len(recv_lists[q]), dtype=torch.float64)
                    if rank < q:
                        if out.numel(): dist.send(out, q)
                        if inc.numel(): dist.recv(inc, q)
                    else:
                        if inc.numel(): dist.recv(inc, q)
                        if out.numel(): dist.send(out, q)
                    y[recv_lists[q]] = inc.numpy()
            else:   # allgatherv via padded all_gather
                m = int(max(bounds[i + 1] - bounds[i] for i in range(world)))
                mine = torch.zeros(m, dtype=torch.float64)
                mine[:hi - lo] = torch.from_numpy(y[lo:hi])
                parts = [torch.zeros(m, dtype=torch.float64) for _ in range(world)]
                dist.all_gather(parts, mine)
                for i in range(world):
                    y[bounds[i]:bounds[i + 1]] = parts[i][:bounds[i + 1] - bounds[i]].numpy()
            x = y
        # gather own slices on rank 0 and compare with the unpartitioned oracle
        m = int(max(bounds[i + 1] - bounds[i] for i in range(world)))
        mine = torch.zeros(m, dtype=torch.float64)
        mine[:hi - lo] = torch.from_numpy(x[lo:hi])
        parts = [torch.zeros(m, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(parts, mine)
        if rank == 0:
            full = np.concatenate([parts[i][:bounds[i + 1] - bounds[i]].numpy() for i in range(world)])
            ref = oracle.iterate(A, x0, K)
            outq.put(("ok", bool(np.array_equal(full, ref)), int(np.isnan(full).sum()),
                   int(sum(len(v) for v in recv_lists.values()))))
        dist.destroy_process_group()
    except Exception as e:   # surface worker failures to the test
        import traceback
        outq.put(("err", repr(e) + traceback.format_exc()))
        raise


@pytest.mark.parametrize("name,exchange", [("lap", "halo"), ("zipf", "halo"), ("banded", "halo"),
                                           ("lap", "allgather"), ("zipf", "allgather")])
def test_two_rank_iterated_spmv_matches_oracle(name, exchange):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    K = 6
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, exchange, K, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=120)
    res = q.get(timeout=5)
    assert res[0] == "ok", res
    _, equal, nans, nghost = res
    assert nans == 0 and equal
    if exchange == "halo" and name == "lap":
        assert nghost == 24          # one grid row of ghosts per neighbour


def _dist_worker(rank, world, port, outq):
    """Each rank holds its OWN (injected) timings of the distribution
    candidates; the agreement the plan makes over NCCL (an elementwise max
    all-reduce of the mean vector, then pepp::dist_argmin) is made here over
    gloo with the library's host rule: every rank must reach the same choice,
    equal to pepp_dist_choose on the stacked [rank][candidate] matrix."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import paper_conf_sc_dastgeerlk12_b200 as pepp
        dist.init_process_group("gloo", rank=rank, world_size=world)
        rng = np.random.default_rng(100 + rank)
        mine = rng.uniform(50, 150, size=6)           # this rank's clock
        t = torch.from_numpy(mine.copy())
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        agreed = t.numpy()
        c_local, ag = pepp.dist_choose(agreed[None, :])
        allm = [torch.zeros(6, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(allm, torch.from_numpy(mine))
        c_ref, ag_ref = pepp.dist_choose(np.stack([m.numpy() for m in allm]))
        outq.put((rank, (c_local, c_ref, bool(np.array_equal(ag, ag_ref)))))
        dist.destroy_process_group()
    except Exception as e:
        import traceback
        outq.put((rank, repr(e) + traceback.format_exc()))


def test_two_rank_distribution_agreement():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_dist_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(30)
    for r in range(2):
        assert isinstance(out[r], tuple), out[r]
        c_local, c_ref, same = out[r]
        assert c_local == c_ref and same
    assert out[0][0] == out[1][0]
