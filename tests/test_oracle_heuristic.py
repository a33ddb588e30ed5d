"""O6 (oracle/heuristic.py, the paper's criteria 1-4, PAPER.md L89-L92 under
reading R25) pinned by hand-derived schedules: each case below was worked out
on paper from the criteria, with fp32-exact utilisations (multiples of 1/8)
so that "kept under 100%" equalities are exact.  A wrong criterion-1 order,
a wrong utilisation column, a strict-vs-equal slip in criterion 2, a missing
memory test (criterion 3), a wrong client limit (criterion 4) or a wrong
fallback each fails one case.  Also: the oracle rank used by O6 is pinned to
oracle.config, and the reported score to oracle.score."""
import numpy as np
import pytest

import oracle
from oracle import heuristic as H
from synth import Query, make_profile, PER_GPU, PER_CLIENT


def _prof(u100, mem=None, u_low=None, levels=(50, 100)):
    n = len(u100)
    prof = make_profile(n, levels=levels, seed=5)
    pct = [int(x) for x in prof.level_pct]
    for i in range(n):
        for li in range(len(pct)):
            prof.sm_util[i, li] = np.float32(u100[i])
        if u_low is not None:
            prof.sm_util[i, pct.index(50)] = np.float32(u_low[i])
        prof.max_mem_mib[i] = 1000 if mem is None else mem[i]
    return prof


U = [0.375, 0.625, 0.125, 0.5]


@pytest.mark.parametrize("g,priority,expect", [
    # order by criterion 1: w2 (0.125), w0 (0.375), w3 (0.5), w1 (0.625)
    # throughput (<= 2 clients): w2, w0 -> GPU0; w3 -> GPU1 (GPU0 full); w1: GPU1 would be 1.125 > 1,
    # no GPU left -> least-utilised GPU with a free client slot = GPU1
    (2, "throughput", [0, 1, 0, 1]),
    # ... with a third GPU w1 opens it
    (3, "throughput", [0, 1, 0, 2]),
    # energy (<= C = 4 clients): w2, w0, w3 -> GPU0 (sum exactly 1.0: kept <= 100 %); w1 -> GPU1
    (2, "energy", [0, 1, 0, 0]),
    # one GPU: everything on it (fallback when 100 % is exceeded)
    (1, "energy", [0, 0, 0, 0]),
])
def test_hand_schedules(g, priority, expect):
    prof = _prof(U)
    q = Query(4, g, 4, (50, 100), PER_GPU, ((1, 1),))
    assert H.canonical(H.schedule(prof, q, priority)) == expect


def test_throughput_one_gpu_two_clients_is_infeasible():
    # criterion 4 (<= 2 clients) on one GPU cannot place 4 workflows
    q = Query(4, 1, 4, (50, 100), PER_GPU, ((1, 1),))
    assert H.schedule(_prof(U), q, "throughput") is None
    assert H.heuristic(_prof(U), q, "throughput") is None


def test_memory_criterion():
    # equal utilisation: queue order.  WarpX 61453 + BerkeleyGW 30157 > 81920
    mem = [61453, 30157, 563, 61453]
    prof = _prof([0.125] * 4, mem=mem)
    q3 = Query(4, 3, 4, (50, 100), PER_GPU, ((1, 1),))
    # w0 -> GPU0; w1 -> GPU1 (memory); w2 -> GPU0; w3 fits nowhere in use -> GPU2
    assert H.canonical(H.schedule(prof, q3, "energy")) == [0, 1, 0, 2]
    q2 = Query(4, 2, 4, (50, 100), PER_GPU, ((1, 1),))
    assert H.schedule(prof, q2, "energy") is None


def test_utilisation_columns():
    # criterion 1 sorts by the 100 % column, criterion 2 sums the column of the
    # level the clients run at (the highest searched level, here 50 %)
    prof = _prof([0.125, 0.25, 0.375], u_low=[0.5, 0.5, 0.25])
    q = Query(3, 2, 3, (50,), PER_GPU, ((1, 1),))
    # order w0, w1, w2 (100 % column); run-level sums: w0 .5, w1 1.0, w2 would be 1.25 -> GPU1
    assert H.canonical(H.schedule(prof, q, "energy")) == [0, 0, 1]
    q100 = Query(3, 2, 3, (50, 100), PER_GPU, ((1, 1),))
    assert H.canonical(H.schedule(prof, q100, "energy")) == [0, 0, 0]   # .125 + .25 + .375 at 100 %


def test_client_limit_respects_c():
    prof = _prof([0.125] * 4)
    q = Query(4, 2, 3, (50, 100), PER_GPU, ((1, 1),))   # C = 3: energy uses at most 3 clients
    assert H.canonical(H.schedule(prof, q, "energy")) == [0, 0, 0, 1]
    q1 = Query(4, 4, 1, (50, 100), PER_GPU, ((1, 1),))  # C = 1: throughput limit min(2, C) = 1
    assert H.canonical(H.schedule(prof, q1, "throughput")) == [0, 1, 2, 3]


@pytest.mark.parametrize("scope", [PER_GPU, PER_CLIENT])
def test_rank_and_score_follow_the_oracle(scope):
    prof = make_profile(6, levels=(25, 50, 75, 100), seed=31)
    q = Query(6, 3, 6, (50, 100), scope, ((1, 1), (1, 0)))
    r = H.heuristic(prof, q, "energy", w=1)
    a, d = oracle.config(q, r["index"])
    assert a == r["rgs"] and all(x == 1 for x in d)
    ok, T, E = oracle.score(prof, q, a, d)
    ts, es = oracle.constants(prof, q)
    assert (ok, T, E) == (r["feasible"], r["T"], r["E"])
    assert r["score64"] == oracle.objective(ts, es, T, E, 1, 0) == ts / T


def test_rank_is_the_inverse_of_config():
    q = Query(5, 3, 3, (25, 100), PER_GPU, ())
    for idx in range(0, oracle.count(q), 7):
        a, d = oracle.config(q, idx)
        assert H.rank(q, a, d) == idx
