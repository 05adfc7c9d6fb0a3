"""Smart containers on the GPU: the paper's Fig. 3 program (P@23511) run with
real components — SpMV (write / read accesses) and a scale (readwrite) —
makes exactly 2 copies of the vector, and every value seen on the host is
the oracle's."""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_sc_dastgeerlk12_b200 as pepp  # noqa: E402

R, W, RW = pepp.ACCESS_READ, pepp.ACCESS_WRITE, pepp.ACCESS_READWRITE


def test_fig3_program_with_spmv_components():
    n = 64
    A = gen.laplacian2d(n)
    N = n * n
    u0 = gen.vector(3, gen.INT8, N)
    with pepp.Plan.from_csr(A) as plan:
        u = pepp.Vector(N, host=u0.copy())
        v0 = pepp.Vector(N)                       # line 2: container created, master copy on host
        w1, w2 = pepp.Vector(N), pepp.Vector(N)
        plan.exec_vec(u, v0)                      # line 4: component writes v0 -> no copy of v0
        assert v0.counters()[:2] == (0, 0)
        ref = oracle.spmv(A, u0)
        assert np.array_equal(v0.host(R), ref)    # line 6: host read -> copy back (1)
        v0.scale(2.0)                             # line 8: readwrite component on the GPU, no copy
        plan.exec_vec(v0, w1)                     # line 10: read-only use, no copy
        plan.exec_vec(v0, w2)                     # line 12: read-only use, no copy
        h = v0.host(W)                            # line 14: host write -> copy back first (2)
        assert np.array_equal(h, 2.0 * ref)
        h2d, d2h, _ = v0.counters()
        assert h2d + d2h == 2 and (h2d, d2h) == (0, 2)
        # the read-only uses computed on the device copy of 2*ref
        assert np.array_equal(w1.host(R), oracle.spmv(A, 2.0 * ref))
        assert np.array_equal(w2.host(R), oracle.spmv(A, 2.0 * ref))
        # u was only read: one copy in, none back
        assert u.counters()[:2] == (1, 0)
        # after the host write the device copy is outdated: the next read copies in
        h[:] = 1.0
        plan.exec_vec(v0, w1)
        assert v0.counters()[:2] == (1, 2)
        assert np.array_equal(w1.host(R), oracle.spmv(A, np.ones(N)))
        for v in (u, v0, w1, w2):
            v.close()


def test_iterated_spmv_through_containers_two_copies():
    """x_{k+1} = A x_k for 16 iterations (integer-exact, P5) with ping-pong containers: the only
    copies are x0 in and the result out."""
    n = 32
    A = gen.laplacian2d(n)
    x0 = gen.vector(3, gen.INT8, n * n)
    with pepp.Plan.from_csr(A) as plan:
        a, b = pepp.Vector(n * n, host=x0.copy()), pepp.Vector(n * n)
        for _ in range(8):
            plan.exec_vec(a, b)
            plan.exec_vec(b, a)
        res = a.host(R)
        assert np.array_equal(res, oracle.iterate(A, x0, 16))
        assert a.counters()[:2] == (1, 1) and b.counters()[:2] == (0, 0)
        a.close(); b.close()


def test_exec_vec_rejects_bad_arguments():
    A = gen.laplacian2d(8)
    with pepp.Plan.from_csr(A) as plan:
        v = pepp.Vector(64)
        with pytest.raises(pepp.PeppError):
            plan.exec_vec(v, v)                      # x and y alias
        short = pepp.Vector(10)
        with pytest.raises(pepp.PeppError):
            plan.exec_vec(short, v)                  # wrong length
        sim = pepp.Vector(64, device=pepp.DEVICE_SIMULATED)
        with pytest.raises(pepp.PeppError):
            plan.exec_vec(sim, v)                    # simulated containers cannot feed kernels


def test_dependencies_across_streams_raw_war():
    """Inter-call parallelism: calls on different streams
    with no explicit synchronisation are ordered by their access modes alone.
    Large vectors make an unordered run visibly wrong."""
    n = 2048
    A = gen.laplacian2d(n)
    N = n * n
    x0 = gen.vector(3, gen.INT8, N)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    with pepp.Plan.from_csr(A) as plan:
        u = pepp.Vector(N, host=x0.copy())
        v, w1, w2, w3 = (pepp.Vector(N) for _ in range(4))
        for _ in range(3):
            plan.exec_vec(u, v, stream=s1)          # v written on s1
            plan.exec_vec(v, w1, stream=s2)         # RAW: s2 must wait for s1
            plan.exec_vec(v, w2, stream=s1)         # read-read: may overlap with the s2 read
            plan.exec_vec(v, w3, stream=s2)
            v.scale(3.0, stream=s1)                 # WAR: must wait for both readers (s1 and s2)
            ref_v = oracle.spmv(A, x0)
            ref_w = oracle.spmv(A, ref_v)
            assert np.array_equal(w1.host(R), ref_w)
            assert np.array_equal(w2.host(R), ref_w)
            assert np.array_equal(w3.host(R), ref_w)
            assert np.array_equal(v.host(R), 3.0 * ref_v)
        for c in (u, v, w1, w2, w3):
            c.close()
