"""Host-side logic of the C-ABI library, CPU only: partitioner, halo ghost
lists, performance history + selection policy (injected "fake clock" times),
context keys. SURVEY.md §4.2 tier T2/T3 host parts."""
from __future__ import annotations

import os
import tempfile

import numpy as np
import pytest

import gen
import oracle
import paper_conf_sc_dastgeerlk12_b200 as pepp


@pytest.mark.parametrize("maker", ["lap", "zipf", "uniform", "banded", "empty_rows"])
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_partition_equals_oracle_definition(maker, P):
    A = {
        "lap": lambda: gen.laplacian2d(40),
        "zipf": lambda: gen.zipf(3000, 3000, seed=46),
        "uniform": lambda: gen.uniform(2000, 2000, 16, seed=42),
        "banded": lambda: gen.banded(1500, 4, seed=100),
        "empty_rows": lambda: gen.CSR(6, 6, np.array([0, 0, 0, 10, 10, 10, 12], dtype=np.int64),
                                      np.zeros(12, np.int32), np.ones(12), 0, 6),
    }[maker]()
    b = pepp.partition_rows(A.row_ptr, P)
    assert np.array_equal(b, oracle.partition_nnz(A, P))
    # with a non-zero `first` (a block of a bigger matrix) the rule is unchanged
    Ar = gen.rebase(A, 1 << 35)
    assert np.array_equal(pepp.partition_rows(Ar.row_ptr, P), b)


def test_partition_laplacian_8192_balanced():
    n = 8192
    rp = np.empty(n * n + 1, dtype=np.int64)
    import ctypes
    gen.lib().gen_laplacian2d_rowptr(n, 0, n * n, rp.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)))
    for P in (2, 4, 8):
        b = pepp.partition_rows(rp, P)
        sizes = np.diff(rp[b])
        assert sizes.max() - sizes.min() <= 10
        assert abs(int(sizes.sum()) - 335_511_552) == 0


@pytest.mark.parametrize("P", [2, 3, 4])
def test_halo_ghosts_match_set_definition(P):
    A = gen.zipf(2500, 2500, seed=7, kmax=60)
    b = pepp.partition_rows(A.row_ptr, P)
    for r in range(P):
        blk = gen.row_block(A, int(b[r]), int(b[r + 1]))
        counts, g = pepp.halo_ghosts(blk.col, P, r, b)
        cols = set(int(c) for c in blk.col)
        expect = sorted(c for c in cols if not (b[r] <= c < b[r + 1]))
        assert g.tolist() == expect
        assert counts[r] == 0 and counts.sum() == len(expect)
        for q in range(P):
            assert counts[q] == sum(1 for c in expect if b[q] <= c < b[q + 1])


def test_halo_laplacian_is_two_grid_rows():
    n, P = 64, 4
    A = gen.laplacian2d(n)
    b = pepp.partition_rows(A.row_ptr, P)
    for r in range(P):
        blk = gen.row_block(A, int(b[r]), int(b[r + 1]))
        counts, g = pepp.halo_ghosts(blk.col, P, r, b)
        # ghosts: n entries below and n above (one grid row each side), contiguous
        if 0 < r < P - 1:
            assert counts[r - 1] == n and counts[r + 1] == n
        assert len(g) == (n if r in (0, P - 1) else 2 * n)


# ------------------------------------------------------------ history ----
def test_history_calibrates_then_exploits_argmin():
    H = pepp.History()
    key = 12345
    times = [5.0, 3.0, 4.0, 3.02]      # fake clock: candidate 1 fastest; 3 within 1 %
    elig = [True] * 4
    order = []
    for _ in range(100):
        c, cal, _ = H.select(key, elig, min_samples=3)
        if not cal:
            break
        order.append(c)
        H.record(key, c, times[c])
    # calibration runs in rounds: every candidate once per round, lowest index
    # first; then refinement rounds (up to 3 x min_samples) for the contenders
    # within 10 % of the best mean: candidates 1 and 3
    assert order == [0, 1, 2, 3] * 3 + [1, 3] * 6
    c, cal, pred = H.select(key, elig, min_samples=3)
    assert (c, cal) == (1, False) and pred == pytest.approx(3.0)
    # candidate 3 is 0.7 % slower: the tie rule keeps the lower index
    assert H.select(key, elig)[0] == 1
    # masking the best one out (disableImpls) picks the next best
    assert H.select(key, [True, False, True, True])[0] == 3
    # other keys are independent (context instances)
    assert H.select(key + 1, elig) == (0, True, 0.0)


def test_history_early_abandonment():
    """A candidate > 4x slower than the best after round 1 is not sampled again."""
    H = pepp.History()
    key = 99
    times = [10.0, 1.0, 300.0, 1.5]
    order = []
    for _ in range(100):
        c, cal, _ = H.select(key, [True] * 4, min_samples=3)
        if not cal:
            break
        order.append(c)
        H.record(key, c, times[c])
    # round 1 samples everyone; candidates 0 (10x) and 2 (300x) are then
    # dropped; no refinement rounds (3 is 50 % slower: the best has no contender)
    assert order == [0, 1, 2, 3, 1, 3, 1, 3]
    assert H.select(key, [True] * 4)[:2] == (1, False)
    assert H.stats(key, 2)[0] == 1 and H.stats(key, 0)[0] == 1


def test_history_tracks_drift_and_welford():
    H = pepp.History()
    xs = [1.0, 2.0, 4.0, 8.0]
    for v in xs:
        H.record(7, 0, v)
    n, m, m2 = H.stats(7, 0)
    assert n == 4 and m == pytest.approx(np.mean(xs)) and m2 / (n - 1) == pytest.approx(np.var(xs, ddof=1))
    # the choice follows the measurements when they change
    for _ in range(3):
        H.record(7, 1, 10.0)
    assert H.select(7, [True, True], 3)[0] == 0
    for _ in range(50):
        H.record(7, 0, 100.0)
    assert H.select(7, [True, True], 3)[0] == 1


def test_history_save_load_merges():
    H = pepp.History()
    for v in (1.0, 3.0):
        H.record(9, 2, v)
    with tempfile.TemporaryDirectory() as d:
        p = os.path.join(d, "h.txt")
        H.save(p)
        G = pepp.History()
        G.record(9, 2, 5.0)
        G.load(p)
        n, m, m2 = G.stats(9, 2)
        assert n == 3 and m == pytest.approx(3.0) and m2 == pytest.approx(np.var([1, 3, 5]) * 3)


def test_history_rejects_bad_input():
    H = pepp.History()
    with pytest.raises(pepp.PeppError):
        H.record(1, 0, float("nan"))
    with pytest.raises(pepp.PeppError):
        H.select(1, [False, False])


def test_context_key_buckets():
    k = pepp.context_key(1 << 20, 1 << 20, 16 << 20, 0.0)
    assert k == pepp.context_key((1 << 20) + 1000, 1 << 20, (16 << 20) + 5000, 0.1)   # same bucket
    assert k != pepp.context_key(1 << 22, 1 << 20, 16 << 20, 0.0)
    assert k != pepp.context_key(1 << 20, 1 << 20, 16 << 20, 3.0)
    assert k != pepp.context_key(1 << 20, 1 << 20, 16 << 20, 0.0, nparts=2)


def test_cold_start_prior_from_nearest_context():
    """Static composition from recorded runs: an unseen context borrows the
    means of the nearest recorded context (bucket distance, same rank count)."""
    H = pepp.History()
    k_small = pepp.context_key(1 << 16, 1 << 16, 16 << 16, 0.0)
    k_big = pepp.context_key(1 << 24, 1 << 24, 16 << 24, 0.0)
    k_other_ranks = pepp.context_key(1 << 20, 1 << 20, 16 << 20, 0.0, nparts=2)
    ids = [10, 20, 30]
    for cid, t in zip(ids, (5.0, 2.0, 9.0)):
        H.record(k_small, cid, t)
    for cid, t in zip(ids, (50.0, 80.0, 20.0)):
        H.record(k_big, cid, t)
    H.record(k_other_ranks, 10, 1.0)
    q = pepp.context_key(1 << 17, 1 << 17, 16 << 17, 0.1)        # nearer to k_small
    prior, src = H.prior(q, ids)
    assert src == k_small and prior.tolist() == [5.0, 2.0, 9.0]
    q2 = pepp.context_key(1 << 23, 1 << 23, 16 << 23, 0.0)       # nearer to k_big
    prior, src = H.prior(q2, ids)
    assert src == k_big and prior.tolist() == [50.0, 80.0, 20.0]
    # ids the neighbour never ran get -1; unknown ids only -> no prior
    prior, _ = H.prior(q, [20, 99])
    assert prior.tolist() == [2.0, -1.0]
    assert H.prior(q, [99]) is None
    # a context with a different rank count never serves as a prior
    q3 = pepp.context_key(1 << 20, 1 << 20, 16 << 20, 0.0, nparts=4)
    assert H.prior(q3, ids) is None


# ------------------------------------------------ distribution choice (a4)
def test_dist_choose_max_over_ranks_then_argmin():
    """P and exchange as timed choices (§8(a) a4, §V-D P@38827): a
    partitioned call lasts as long as its slowest rank, so candidate d's
    agreed time is the max over ranks; the choice is its argmin (A10 tie
    rule). Injected times: rank 1 is slow on candidate 0, so candidate 2
    (never the fastest on either rank alone) wins."""
    means = [[10.0, 30.0, 12.0, 50.0],
             [25.0, 11.0, 13.0, 40.0]]
    c, agreed = pepp.dist_choose(means)
    assert list(agreed) == [25.0, 30.0, 13.0, 50.0]
    assert c == 2
    # eligibility (e.g. REPLICATED calls: allgather candidates only)
    c, _ = pepp.dist_choose(means, eligible=[True, True, False, True])
    assert c == 0
    # ties within 1 % go to the lower index; 2 % apart does not tie
    c, _ = pepp.dist_choose([[100.0, 99.5]])
    assert c == 0
    c, _ = pepp.dist_choose([[100.0, 98.0]])
    assert c == 1
    # untimed (0) candidates are skipped
    c, _ = pepp.dist_choose([[0.0, 5.0], [0.0, 6.0]])
    assert c == 1


def test_dist_choose_rejects_bad_input():
    with pytest.raises(pepp.PeppError):
        pepp.dist_choose([[1.0, float("nan")]])
    with pytest.raises(pepp.PeppError):
        pepp.dist_choose([[-1.0, 2.0]])
    with pytest.raises(pepp.PeppError):
        pepp.dist_choose([[1.0, 2.0]], eligible=[False, False])


def test_global_switches_from_environment():
    """The paper's global tool switches (disableImpls P@16687, useHistoryModels
    P@28058) as environment defaults of pepp_spmv_opts_default; explicit
    options set afterwards win (the per-component form)."""
    import subprocess
    import sys
    code = ("import ctypes, paper_conf_sc_dastgeerlk12_b200._capi as C; o = C.OPTS_T(); "
            "C.lib().pepp_spmv_opts_default(ctypes.byref(o)); "
            "print(o.variant_mask, o.use_history, (o.history_path or b'').decode())")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    base = {k: v for k, v in os.environ.items() if not k.startswith("PEPP_")}
    out = subprocess.run([sys.executable, "-c", code], env=base, capture_output=True, text=True, cwd=root)
    assert out.stdout.split() == ["0", "1"], out.stderr
    env = dict(base, PEPP_VARIANT="sell,merge_path", PEPP_USE_HISTORY="0", PEPP_HISTORY_PATH="/tmp/h.txt")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, cwd=root)
    assert out.stdout.split() == [str((1 << pepp.V_SELL) | (1 << pepp.V_MERGE_PATH)), "0", "/tmp/h.txt"], out.stderr
    env = dict(base, PEPP_VARIANT="nonsense")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, cwd=root)
    assert out.stdout.split()[0] == "0"
