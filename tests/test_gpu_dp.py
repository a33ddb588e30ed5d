"""GPU subset-DP front (sched_front_dp, dp_front.cu) against
the oracle: the full enumeration O1 on small PER_CLIENT / PER_GPU spaces and
the O3/O4 certificates (front values, per-weight optimum, bitwise); every
witness configuration re-scored by the oracle to its point; and the literal
per-client c4 (4.05e19 configurations) run with its witnesses re-scored."""
import dataclasses

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, Query, PER_CLIENT, PER_GPU

pytestmark = pytest.mark.gpu

W = ((1, 1), (2, 1), (1, 0), (0, 1), (1, 3))


def _witness_ok(prof, q, pt):
    n = q.n
    rgs = [int(pt.group_of[i]) for i in range(n)]
    lv = [int(pt.level_of[i]) for i in range(n)]
    digits = lv if q.scope == PER_CLIENT else [lv[rgs.index(g)] for g in range(max(rgs) + 1)]
    ok, T, E = oracle.score(prof, q, rgs, digits)
    return ok and T == pt.makespan_s and E == pt.energy_j


@pytest.mark.parametrize("n,g,c,levels,scope,seed", [
    (5, 2, 3, (25, 50, 75, 100), PER_CLIENT, 700), (6, 3, 3, (50, 100), PER_CLIENT, 701),
    (7, 3, 7, (25, 50, 75, 100), PER_CLIENT, 702), (6, 4, 2, (50, 100), PER_CLIENT, 703),
    (8, 3, 3, (50, 100), PER_CLIENT, 707), (9, 4, 4, (25, 50, 75, 100), PER_GPU, 708),
    (8, 8, 8, (100,), PER_GPU, 709),
])
def test_dp_front_vs_enumeration(n, g, c, levels, scope, seed):
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, levels, scope, W, True)
    ref = oracle.search(prof, q)
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    assert st["kernel_path"] == 4
    assert [(p.makespan_s, p.energy_j) for p in front] == [(T, E) for _, T, E in ref["pareto"]]
    for w in range(len(W)):
        assert best[w].score64 == ref["best"][w][1]
    for p in list(front) + list(best):
        assert _witness_ok(prof, q, p)


@pytest.mark.parametrize("n,g,c,seed", [(11, 4, 4, 801), (12, 6, 3, 802)])
def test_dp_front_vs_client_certificate(n, g, c, seed):
    """PER_CLIENT spaces too large for O1 (1e10+ configurations) against the
    O4 certificate."""
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed, g=g, c=c)
    q = Query(n, g, c, (25, 50, 75, 100), PER_CLIENT, W, True)
    cert = oracle.dp_certificate(prof, q)
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    assert [(p.makespan_s, p.energy_j) for p in front] == cert["front"]
    assert [b.score64 for b in best] == cert["best"]
    for p in front:
        assert _witness_ok(prof, q, p)


def test_dp_front_c4_per_gpu_equals_certificate():
    """The PER_GPU c4 front by the device DP == the stored O3 certificate."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c4_certificate.json")))
    prof, q = config("c4")
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    assert [[p.makespan_s.hex(), p.energy_j.hex()] for p in front] == g["front_T_E"]
    assert [b.score64.hex() for b in best] == g["best_score64"]


def test_dp_front_c4_literal_per_client():
    """Literal per-client c4: 4.05e19 configurations.  Every front point's
    witness is re-scored by the oracle; the per-client optimum can only be at
    least the per-GPU one (PER_GPU is a subset of PER_CLIENT)."""
    prof, q = config("c4")
    qc = dataclasses.replace(q, scope=PER_CLIENT)
    rc, best, front, st = S.Scheduler(prof).front_dp(qc)
    assert rc == S.sched.SCHED_OK and len(front) > 0
    for p in list(front) + list(best):
        assert _witness_ok(prof, qc, p)
    _, bg, _, _ = S.Scheduler(prof).front_dp(q)
    for w in range(len(q.weights)):
        assert best[w].score64 >= bg[w].score64
    print("c4 per-client:", st["search_ms"], "ms;", len(front), "front points;",
          [b.score64 for b in best], "vs per-GPU", [b.score64 for b in bg])


@pytest.mark.parametrize("n", [13, 14, 16])
def test_dp_front_c4_client_prefix_golden(n):
    """Literal per-client reading on the c4 profile: the first 13 / 14
    workflows and the whole c4 queue (n = 16: 4.05e19 configurations, the
    north star's "per-client active-thread percentage"), G = 8, 4
    levels per client: front values and optimum per weight bitwise equal to
    the stored O4 certificate (tests/golden, written by
    `python -m oracle.make_certificates client n [procs]`; n = 16 took 75
    minutes on 7 host processes)."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", f"c4_client_n{n}_certificate.json")))
    prof, q = config("c4")
    q = dataclasses.replace(q, n=n, scope=PER_CLIENT, weights=tuple(tuple(w) for w in g["weights"]))
    p = prof.subset(n)
    rc, best, front, st = S.Scheduler(p).front_dp(q)
    assert rc == S.sched.SCHED_OK and st["kernel_path"] == 4
    assert [[x.makespan_s.hex(), x.energy_j.hex()] for x in front] == g["front_T_E"]
    assert [b.score64.hex() for b in best] == g["best_score64"]
    for x in list(front) + list(best):
        assert _witness_ok(p, q, x)


def test_dp_front_c5_equals_certificate():
    """c5 (20 workflows, 8 GPUs, <= 3 clients per GPU, 6.0e11 configurations):
    the device DP front and the 7-weight sweep optimum equal the stored O3
    certificate bitwise (tests/golden/c5_certificate.json)."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c5_certificate.json")))
    prof, q = config("c5")
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    assert rc == S.sched.SCHED_OK and st["kernel_path"] == 4
    assert [[p.makespan_s.hex(), p.energy_j.hex()] for p in front] == g["front_T_E"]
    assert [b.score64.hex() for b in best] == g["best_score64"]
    for p in list(front) + list(best):
        assert _witness_ok(prof, q, p)
    print("c5 DP:", st["total_ms"], "ms")


def _canon(lab):
    m = {}
    return [m.setdefault(x, len(m)) for x in lab]


def test_dp_front_c4_literal_per_client_no_better_neighbour_or_sample():
    """Literal per-client c4 (n = 16: no full oracle, DESIGN.md 'parity
    partial') -- properties every correct front has at any size, checked with
    the oracle's fp64 scorer: no configuration one move away from a witness
    (one client's level changed, or one client moved to another / a new
    group) and none of 20000 seeded random configurations strictly dominates
    a front point or beats a per-weight optimum.  Catches a DP that drops a
    level combination, a group split or a subset state."""
    import random
    prof, q = config("c4")
    qc = dataclasses.replace(q, scope=PER_CLIENT)
    rc, best, front, st = S.Scheduler(prof).front_dp(qc)
    assert rc == S.sched.SCHED_OK and len(front) > 0
    pts = [(p.makespan_s, p.energy_j) for p in front]
    ts, es = oracle.constants(prof, qc)
    n, L, G = qc.n, len(qc.levels), qc.g

    def check(rgs, digits):
        ok, T, E = oracle.score(prof, qc, rgs, digits)
        if not ok:
            return 0
        for (pt, pe) in pts:
            assert not (T <= pt and E <= pe and (T < pt or E < pe)), (rgs, digits, T, E, pt, pe)
        for w, (a, b) in enumerate(qc.weights):
            assert oracle.objective(ts, es, T, E, a, b) <= best[w].score64
        return 1

    nfeas = 0
    for p in list(front) + list(best):
        rgs = [int(p.group_of[i]) for i in range(n)]
        lv = [int(p.level_of[i]) for i in range(n)]
        k = max(rgs) + 1
        for i in range(n):
            for d in range(L):
                if d != lv[i]:
                    nfeas += check(rgs, lv[:i] + [d] + lv[i + 1:])
            for gnew in range(min(k + 1, G)):
                if gnew != rgs[i]:
                    lab = rgs[:i] + [gnew] + rgs[i + 1:]
                    nfeas += check(_canon(lab), lv)
    rnd = random.Random(16)
    for _ in range(20000):
        lab = [rnd.randrange(G) for _ in range(n)]
        nfeas += check(_canon(lab), [rnd.randrange(L) for _ in range(n)])
    assert nfeas > 10000


@pytest.mark.parametrize("model", [1, 5])
@pytest.mark.parametrize("n,g,c,levels,scope,seed", [
    (6, 3, 3, (50, 100), PER_CLIENT, 711), (7, 3, 7, (25, 50, 75, 100), PER_CLIENT, 712),
    (9, 4, 4, (25, 50, 75, 100), PER_GPU, 713), (8, 8, 8, (100,), PER_GPU, 714),
])
def test_dp_front_count_idle_vs_enumeration(model, n, g, c, levels, scope, seed):
    """COUNT_IDLE (R26: E = G P_s T + sum D_g; round 2: the DP adds up D_g and
    applies the idle term to the whole-set front) alone and with POWER_CAP:
    front values, per-weight optimum and witnesses equal the oracle's full
    enumeration."""
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, levels, scope, W, True, model=model, power_cap=140.0)
    ref = oracle.search(prof, q)
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    assert st["kernel_path"] == 4
    assert [(p.makespan_s, p.energy_j) for p in front] == [(T, E) for _, T, E in ref["pareto"]]
    for w in range(len(W)):
        assert best[w].score64 == ref["best"][w][1]
    for p in list(front) + list(best):
        assert _witness_ok(prof, q, p)
