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


def test_bench_two_ranks_one_gpu():
    sys.path.insert(0, HERE)
    from test_gpu_partitioned import _build_fake
    env = dict(os.environ, PEPP_NCCL_LIB=_build_fake(), PEPP_BENCH_ONE_DEVICE="1", PEPP_BENCH_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1",
           "--warmup", "3", "--workload", "lap2048", "--no-sweep"]
    out = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 1 and d["value"] > 0
    # halo pushed by the fused boundary kernel into the peer's buffer (PEPP_X_P2P, CUDA IPC on one device)
    assert d["config"]["exchange"].startswith("p2p")
    # rank 0's block sends its last grid row: interior kernel + the fused tail/push kernel per SpMV
    assert d["plan"]["overlap"] == 1 and d["plan"]["overlap_head"] == 0 and d["plan"]["overlap_tail"] == 2048
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] >= 200
    assert "launch_includes" in d["roofline"]
    assert d["cpu_baseline"] is None          # rank 0 at N = 1 only
