"""bench.py's multi-rank path on ONE GPU: torch.distributed.run with two
ranks, gloo for torch.distributed, the library pointed at the NCCL stand-in
(tests/support/fake_nccl.c) and every rank on device 0 (test-only knobs
PEPP_BENCH_ONE_DEVICE / PEPP_BENCH_DIST_BACKEND). Checks the contract, not
the numbers: exactly one JSON line from rank 0, n_gpus = 2, the fused
peer-memory halo (PEPP_X_P2P) in use, the max-over-ranks timing and the e2e leg present."""
from __future__ import annotations

import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)


def _port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("launch,fault", [("torchrun", False), ("self", False), ("self", True)])
def test_bench_two_ranks_one_gpu(launch, fault):
    """launch = torchrun: the driver's command line; self: `python bench.py
    --gpus 2` with no WORLD_SIZE re-executes itself under
    torch.distributed.run. fault: rank 1's CUDA-IPC export is made to fail
    (PEPP_FAULT_P2P_EXPORT=1): every rank gets the agreed error and the bench
    falls back to the NCCL halo (reported in run.p2p_fallback)."""
    sys.path.insert(0, HERE)
    from test_gpu_partitioned import _build_fake
    # PEPP_FAKE_NCCL_BOX_MB: the distribution candidate P' = 1 ships rank 1's
    # block (~120 MB of lap2048) to rank 0 in one message at plan time
    env = dict(os.environ, PEPP_NCCL_LIB=_build_fake(), PEPP_BENCH_ONE_DEVICE="1", PEPP_BENCH_DIST_BACKEND="gloo",
               PEPP_FAKE_NCCL_BOX_MB="160")
    env.pop("WORLD_SIZE", None)
    if fault:
        env["PEPP_FAULT_P2P_EXPORT"] = "1"
    tail = [os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1", "--warmup", "3", "--workload", "lap2048",
            "--no-sweep"]
    if launch == "torchrun":
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
               "127.0.0.1", "--master-port", str(_port()), *tail]
    else:
        cmd = [sys.executable, *tail]
    out = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 1 and d["value"] > 0
    # the distribution choice (row a4): every (P', exchange) candidate timed and agreed
    dist = d["run"]["distribution"]
    assert dist and {(c["nparts"], c["exchange"]) for c in dist} >= {(2, "halo"), (2, "allgather"), (1, "halo"),
                                                                     (1, "allgather")}
    if not fault:
        # the fused push was registered and timed as a candidate too
        assert d["run"]["p2p_fallback"] is None and any(c["exchange"] == "p2p" for c in dist)
    else:
        assert not d["run"]["exchange"].startswith("p2p") and "PEPP_E_CUDA" in d["run"]["p2p_fallback"], d["run"]
        assert not any(c["exchange"] == "p2p" for c in dist)
    # rank 0's block sends its last grid row (head / interior / tail split)
    assert d["plan"]["overlap"] == 1 and d["plan"]["overlap_head"] == 0 and d["plan"]["overlap_tail"] == 2048
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] >= 100
    assert d["cpu_baseline"] is None          # rank 0 at N = 1 only
    assert d["configs"] is None               # the config 1-3 legs run at N = 1 only
