"""Smart containers (paper §IV-D), CPU only: the copy
protocol runs on simulated vectors (state machine + counters, no CUDA) and
is pinned to the paper's Fig. 3 numbers (tests/golden/paper_constants.json):
the Fig. 3 program makes 2 copies with containers, 7 when every call copies
its operand in and out."""
from __future__ import annotations

import json
import os

import pytest

import paper_conf_sc_dastgeerlk12_b200 as pepp

R, W, RW = pepp.ACCESS_READ, pepp.ACCESS_WRITE, pepp.ACCESS_READWRITE
GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_constants.json")))["fig3_copy_operations"]

# Fig. 3's program after the container is created (P@23793-24990)
FIG3 = [("call", W), ("host", R), ("call", RW), ("call", R), ("call", R), ("host", W)]


def _run(v, prog):
    states = []
    for kind, mode in prog:
        if kind == "call":
            v.device(mode, stream=False)
            v.release(stream=False)
        else:
            v.host(mode)
        states.append(v.state())
    return states


def test_fig3_two_copies_with_containers():
    v = pepp.Vector(1000, device=pepp.DEVICE_SIMULATED)
    assert v.state() == (True, False)            # master copy on the host
    states = _run(v, FIG3)
    h2d, d2h, nbytes = v.counters()
    assert h2d + d2h == GOLD["with_containers"] == 2
    assert (h2d, d2h) == (0, 2)                   # both copies are device -> host
    assert nbytes == 2 * 1000 * 8
    # the state walk the paper describes line by line
    assert states == [
        (False, True),   # line 4: write on the GPU, no copy; master outdated
        (True, True),    # line 6: host read copies back; device copy stays valid
        (False, True),   # line 8: readwrite on the GPU uses the device copy; master outdated
        (False, True),   # line 10: read, no copy
        (False, True),   # line 12: read, no copy
        (True, False),   # line 14: host write copies back first; device copy outdated
    ]


def _per_call_copies(prog):
    """The comparison the paper draws: every component call copies what it
    reads in and everything back out (considering each call independently)."""
    n = 0
    for kind, mode in prog:
        if kind == "call":
            n += (1 if mode & R else 0) + 1
    return n


def test_fig3_seven_copies_when_each_call_copies():
    assert _per_call_copies(FIG3) == GOLD["per_call_copying"] == 7


def test_protocol_rules():
    v = pepp.Vector(10, device=pepp.DEVICE_SIMULATED)
    v.device(R, stream=False)                      # read needs the data: one copy in
    assert v.counters()[:2] == (1, 0) and v.state() == (True, True)
    v.device(R, stream=False)                      # still valid: nothing
    v.host(R)                                      # host valid: nothing
    assert v.counters()[:2] == (1, 0)
    v.host(W)                                      # host write: device outdated
    assert v.state() == (True, False)
    v.device(W, stream=False)                      # write-only: no copy in
    assert v.counters()[:2] == (1, 0) and v.state() == (False, True)
    v.device(RW, stream=False)                     # device copy valid: nothing
    v.host(RW)                                     # copy back once
    assert v.counters()[:2] == (1, 1) and v.state() == (True, False)
    v.device(RW, stream=False)                     # copy in (device outdated), then master outdated
    assert v.counters()[:2] == (2, 1) and v.state() == (False, True)
    with pytest.raises(pepp.PeppError):
        v.device(0, stream=False)
