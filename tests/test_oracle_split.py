"""O5 (oracle/split.py, R29) pinned by: the
divisor-count closed form and the rank order of split vectors, a hand-built
expanded profile, the all-ones split reducing to the plain search, an
independent brute-force search over every split (O2 scorer on a separately
built expansion), and closed forms for the interference-free limit."""
import dataclasses
import math

import numpy as np
import pytest

import oracle
import oracle.brute as br
from oracle import split as O5
from synth import make_profile, Query, PER_CLIENT, PER_GPU


def _ndiv(k):   # divisor function from the prime factorisation
    r, p = 1, 2
    while p * p <= k:
        e = 0
        while k % p == 0:
            k //= p
            e += 1
        r *= e + 1
        p += 1
    return r * (2 if k > 1 else 1)


@pytest.mark.parametrize("tasks", [(1,), (4,), (2, 3), (12, 1, 6), (4, 4, 4, 4), (7, 9, 30)])
def test_split_count_is_divisor_product(tasks):
    sv = O5.split_vectors(tasks)
    assert len(sv) == math.prod(_ndiv(k) for k in tasks)
    assert sv == sorted(sv) and len(set(sv)) == len(sv)
    assert all(k % p == 0 for v in sv for p, k in zip(v, tasks))


def test_split_order_and_cap_literal():
    assert O5.split_vectors((2, 3)) == [(1, 1), (1, 3), (2, 1), (2, 3)]
    assert O5.split_vectors((4, 6), max_split=(2, 3)) == [(1, 1), (1, 2), (1, 3), (2, 1), (2, 2), (2, 3)]


def test_expanded_profile_by_hand():
    prof = make_profile(2, levels=(50, 100), seed=3)
    ep = O5.expand_profile(prof, 2, (4, 3), (2, 1))
    assert ep.n_workflows == 3
    for l in range(2):
        # clients 0, 1 of workflow 0 run 2 of its 4 tasks; client 2 = workflow 1 whole
        assert ep.solo_time_s[0, l] == np.float32(float(prof.solo_time_s[0, l]) * 2 / 4)
        assert ep.solo_time_s[1, l] == ep.solo_time_s[0, l]
        assert ep.solo_time_s[2, l] == prof.solo_time_s[1, l]
        assert ep.solo_power_w[1, l] == prof.solo_power_w[0, l] and ep.sm_util[2, l] == prof.sm_util[1, l]
        for m in range(2):
            assert ep.corun_slowdown[0, l, 1, m] == prof.corun_slowdown[0, l, 0, m]   # siblings: diagonal
            assert ep.corun_slowdown[1, l, 2, m] == prof.corun_slowdown[0, l, 1, m]
            assert ep.corun_slowdown[2, l, 0, m] == prof.corun_slowdown[1, l, 0, m]
    assert list(ep.max_mem_mib) == [prof.max_mem_mib[0]] * 2 + [prof.max_mem_mib[1]]
    assert prof.corun_slowdown[0, 0, 0, 0] > 0          # synth draws a self co-run slowdown


def test_all_ones_split_is_plain_search():
    prof = make_profile(4, levels=(50, 100), seed=1)
    q = Query(4, 2, 4, (50, 100), PER_CLIENT, ((1, 0), (0, 1), (1, 1), (2, 1)))
    r = O5.search_splits(prof, q, (1, 1, 1, 1))
    ref = oracle.search(prof, q)
    assert r["splits"] == [(1, 1, 1, 1)]
    assert [(b[2], b[0]) for b in r["best"]] == [(x[0], x[1]) for x in ref["best"]]
    assert [(T, E, i) for T, E, _, i in r["pareto"]] == [(T, E, i) for i, T, E in ref["pareto"]]


def _brute_splits(prof, q, tasks):
    """Independent: expansion by np.repeat, O2 scores, F with the unsplit baselines."""
    pct = [int(x) for x in prof.level_pct]
    lev = [pct.index(v) for v in q.levels]
    l100 = pct.index(100)
    t100 = [float(prof.solo_time_s[i, l100]) for i in range(q.n)]
    p100 = [float(prof.solo_power_w[i, l100]) for i in range(q.n)]
    ps = float(prof.static_power_w)
    ts = br.t_seq(t100, q.g)
    es = br.e_seq(p100, t100, ps)
    chosen = [[p for p in range(1, k + 1) if k % p == 0] for k in tasks[:q.n]]
    allpts, best = [], [None] * len(q.weights)
    rank = 0
    def rec(i, sv):
        nonlocal rank
        if i == q.n:
            own = np.repeat(np.arange(q.n), sv)
            s = np.array([tasks[o] // sv[o] for o in own], float)
            K = np.array([tasks[o] for o in own], float)
            t = (prof.solo_time_s[own].astype(float) * s[:, None] / K[:, None]).astype(np.float32)
            ep = dataclasses.replace(prof, solo_time_s=t, solo_power_w=prof.solo_power_w[own],
                                     sm_util=prof.sm_util[own], bw_util=prof.bw_util[own],
                                     max_mem_mib=prof.max_mem_mib[own],
                                     corun_slowdown=np.ascontiguousarray(prof.corun_slowdown[own][:, :, own]))
            m = len(own)
            for idx, (rgs, dig) in enumerate(br.space(m, q.g, min(q.c, m), len(q.levels), q.scope)):
                lvp = [lev[dig[a] if q.scope == PER_CLIENT else dig[rgs[a]]] for a in range(m)]
                ok, T, E = br.score(ep, m, rgs, lvp)
                if not ok:
                    continue
                allpts.append((T, E, rank, idx))
                for w, (a, b) in enumerate(q.weights):
                    F = oracle.objective(ts, es, T, E, a, b)
                    if best[w] is None or F > best[w][0]:
                        best[w] = (F, rank, idx, T, E)
            rank += 1
            return
        for p in chosen[i]:
            rec(i + 1, sv + [p])
    rec(0, [])
    front = [x for x in allpts
             if not any(y[0] <= x[0] and y[1] <= x[1] and (y[0] < x[0] or y[1] < x[1]) for y in allpts)]
    uniq = {}
    for x in sorted(front):
        uniq.setdefault((x[0], x[1]), x)
    return best, sorted(uniq.values()), ts, es


@pytest.mark.parametrize("n,tasks,g,c,levels,scope,seed", [
    (2, (2, 2), 2, 4, (50, 100), PER_CLIENT, 0),
    (2, (4, 2), 2, 2, (100,), PER_GPU, 1),
    (3, (2, 1, 3), 2, 3, (50, 100), PER_GPU, 2),
    (3, (2, 2, 1), 3, 5, (25, 100), PER_CLIENT, 3),
])
def test_split_search_vs_brute(n, tasks, g, c, levels, scope, seed):
    prof = make_profile(n, levels=levels, seed=seed)
    q = Query(n, g, c, levels, scope, ((1, 0), (0, 1), (1, 1), (2, 1), (1, 2)))
    r = O5.search_splits(prof, q, tasks)
    best, front, ts, es = _brute_splits(prof, q, tasks)
    assert (r["tseq"], r["eseq"]) == (ts, es)
    assert r["best"] == best
    assert r["pareto"] == front


def test_interference_free_limit_closed_form():
    """d = 0, utilisations tiny, G >= total tasks, one level: splitting every
    workflow into single tasks gives T = max_i t_i / K_i and, all clients on
    one GPU, E = P_s T + sum_i (p_i - P_s) t_i (up to the fp32 rounding of
    the client times): X, Y of the optimum in closed form."""
    prof = make_profile(3, levels=(100,), seed=5)
    prof.corun_slowdown[:] = 0.0
    prof.sm_util[:] = 0.01
    prof.bw_util[:] = 0.01
    tasks = (4, 2, 6)
    q = Query(3, 12, 12, (100,), PER_GPU, ((1, 0), (0, 1)), True)
    r = O5.search_splits(prof, q, tasks)
    t = prof.solo_time_s[:, 0].astype(float)
    p = prof.solo_power_w[:, 0].astype(float)
    ps = float(prof.static_power_w)
    tseq = max(t)                                   # G >= n: list schedule = max t
    eseq = float(sum(p * t))
    Tbest = max(t[i] / tasks[i] for i in range(3))
    assert r["best"][0][3] == pytest.approx(Tbest, rel=1e-6)
    assert r["best"][0][0] == pytest.approx(tseq / Tbest, rel=1e-6)
    Ebest = ps * Tbest + float(sum((p - ps) * t))
    assert r["best"][1][0] == pytest.approx(eseq / Ebest, rel=1e-6)
    assert r["splits"][r["best"][1][1]] == tasks
