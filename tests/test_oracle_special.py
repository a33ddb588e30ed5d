"""Pins of the oracle's score against closed forms, special cases and the paper's numbers.

Each test names the mistake it would catch.
"""
import itertools
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import oracle.brute as br
from synth import make_profile, table_iii_combo1, Query, PER_CLIENT, PER_GPU, TABLE_II

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _q(n, g, c, levels, scope, weights=((1, 0), (0, 1), (1, 1), (2, 1))):
    return Query(n, g, c, levels, scope, weights, True)


def test_e_seq_table_ii_combo1():
    """E_seq = sum iters x Energy (PAPER.md L96 sequential energy; Table II
    L101/L110; Table III combo 1 L145): 5*5407.36 + 3*29390.48 = 115208.24 J.
    Catches: dynamic/static split wrongly applied to the sequential baseline."""
    prof = table_iii_combo1()
    ts, es = oracle.constants(prof, _q(2, 2, 2, (100,), PER_GPU))
    assert es == pytest.approx(115208.24, rel=1e-6)
    g = json.load(open(os.path.join(GOLD, "worked_example_combo1.json")))
    assert es == pytest.approx(g["E_seq_J"], rel=1e-6)


def test_t_seq_list_schedule():
    """G = 1 -> T_seq = sum t; G >= N -> max t; G=2 queue order list schedule
    (PAPER.md L96 'individually on GPUs in queue order').  Catches: wrong
    baseline (e.g. sum on every G, or LPT order)."""
    prof = make_profile(5, levels=(100,), seed=5)
    t = [float(x) for x in prof.solo_time_s[:, 0]]
    assert oracle.constants(prof, _q(5, 1, 5, (100,), PER_GPU))[0] == pytest.approx(sum(t), rel=1e-15)
    assert oracle.constants(prof, _q(5, 5, 5, (100,), PER_GPU))[0] == max(t)
    fin = [0.0, 0.0]
    for x in t:
        j = 0 if fin[0] <= fin[1] else 1
        fin[j] += x
    assert oracle.constants(prof, _q(5, 2, 5, (100,), PER_GPU))[0] == pytest.approx(max(fin), rel=1e-15)


def test_singletons_at_full_level_are_sequential():
    """N <= G, every workflow alone at 100%: tau = t (sigma = 1, c = 1 since
    u, bw <= 1), T = max t = T_seq -> X = 1; E = sum (P_s t + (p-P_s) t) =
    E_seq -> Y = 1.  Catches: sign of dyn, c_g floor missing, idle energy."""
    for seed in range(5):
        n = 5
        prof = make_profile(n, levels=(50, 100), seed=seed)
        q = _q(n, n, n, (50, 100), PER_GPU)
        ts, es = oracle.constants(prof, q)
        ok, T, E = oracle.score(prof, q, list(range(n)), [1] * n)
        assert ok
        assert ts / T == 1.0
        assert es / E == pytest.approx(1.0, abs=1e-12)


def test_no_interference_low_util_group():
    """d = 0 and sum u, sum bw <= 1 -> tau_i = t_i, T_g = max t, E_g =
    P_s max t + sum dyn.  Catches: stretch applied below 100%, d diagonal used."""
    prof = make_profile(4, levels=(100,), seed=9, archetypes=[0, 3, 5, 1])
    prof.corun_slowdown[:] = 0.0
    prof.corun_slowdown[0, 0, 0, 0] = 123.0   # diagonal must be ignored
    q = _q(4, 1, 4, (100,), PER_GPU)
    assert float(prof.sm_util[:, 0].sum()) <= 1.0 and float(prof.bw_util[:, 0].sum()) <= 1.0
    ok, T, E = oracle.score(prof, q, [0, 0, 0, 0], [0])
    t = prof.solo_time_s[:, 0].astype(float)
    p = prof.solo_power_w[:, 0].astype(float)
    assert T == max(t)
    assert E == pytest.approx(60.0 * max(t) + sum((p - 60.0) * t), rel=1e-13)


def _fr(x):
    return Fraction(float(np.float32(x)))


def test_worked_example_combo1_exact_rationals():
    """Table III combo 1 with d_AL = 0.05, d_LA = 0.10, one
    level.  Expected values evaluated in exact rational arithmetic from the
    fp32 inputs (independent of fp64 rounding order) and checked against
    the hand-computed numbers in tests/golden/worked_example_combo1.json.
    Catches: transposed d (A's slowdown must use d[A][L]), wrong c_g, wrong
    objective exponents."""
    g = json.load(open(os.path.join(GOLD, "worked_example_combo1.json")))
    prof = table_iii_combo1((0.05, 0.10))
    tA, tL = _fr(prof.solo_time_s[0, 0]), _fr(prof.solo_time_s[1, 0])
    pA, pL = _fr(prof.solo_power_w[0, 0]), _fr(prof.solo_power_w[1, 0])
    uA, uL = _fr(prof.sm_util[0, 0]), _fr(prof.sm_util[1, 0])
    bA, bL = _fr(prof.bw_util[0, 0]), _fr(prof.bw_util[1, 0])
    dAL, dLA = _fr(0.05), _fr(0.10)
    Ps = Fraction(60)
    cg = max(Fraction(1), uA + uL, bA + bL)
    T = max(tA * (1 + dAL) * cg, tL * (1 + dLA) * cg)
    E = Ps * T + (pA - Ps) * tA + (pL - Ps) * tL
    Eseq = pA * tA + pL * tL
    for G in (1, 2):
        q = Query(2, G, 2, (100,), PER_GPU, ((1, 0), (0, 1), (1, 1), (2, 1)), True)
        ts, es = oracle.constants(prof, q)
        Tseq = tA + tL if G == 1 else max(tA, tL)
        assert ts == pytest.approx(float(Tseq), rel=1e-15)
        assert es == pytest.approx(float(Eseq), rel=1e-15)
        ok, To, Eo = oracle.score(prof, q, [0, 0], [0])
        assert ok and To == pytest.approx(float(T), rel=1e-14) and Eo == pytest.approx(float(E), rel=1e-14)
        X, Y = Tseq / T, Eseq / E
        gold = g["G%d" % G]
        assert float(X) == pytest.approx(gold["X_together"], rel=1e-6)
        assert float(Y) == pytest.approx(g["Y_together"], rel=1e-6)
        r = oracle.search(prof, q)
        if G == 1:
            assert r["nconfigs"] == 1 and [b[0] for b in r["best"]] == [0, 0, 0, 0]
            assert r["best"][2][1] == pytest.approx(float(X * Y), rel=1e-14)
            assert r["best"][3][1] == pytest.approx(float(X * X * Y), rel=1e-14)
        else:
            # idx 0 = {A,L} together, idx 1 = separate (X = 1, Y = 1)
            assert r["nconfigs"] == 2
            assert [b[0] for b in r["best"]] == gold["best_idx_per_weight"]
            assert [p[0] for p in r["pareto"]] == gold["pareto_idx_by_X_desc"]


def _group_T(prof, members, lv):
    """Group makespan written out for the min-makespan DP (pins the SEARCH)."""
    u = sum(float(prof.sm_util[i, lv]) for i in members)
    b = sum(float(prof.bw_util[i, lv]) for i in members)
    c = max(1.0, u, b)
    T = 0.0
    for i in members:
        s = 1.0 + sum(float(prof.corun_slowdown[i, lv, j, lv]) for j in members if j != i)
        T = max(T, float(prof.solo_time_s[i, lv]) * s * c)
    return T


def test_min_makespan_subset_dp():
    """Throughput-only optimum (weight (1,0)) = T_seq / min T, where min T is
    computed by an independent subset DP over groups (PER_GPU: best level per
    group).  Catches: enumeration that misses partitions or level vectors."""
    for seed, (n, g, c) in enumerate([(6, 3, 3), (7, 3, 7), (7, 4, 2)]):
        prof = make_profile(n, levels=(25, 50, 100), seed=40 + seed)
        q = Query(n, g, c, (25, 50, 100), PER_GPU, ((1, 0),), False)
        r = oracle.search(prof, q)
        full = (1 << n) - 1
        grpT = {}
        for S in range(1, full + 1):
            mem = [i for i in range(n) if S >> i & 1]
            if len(mem) > c or sum(int(prof.max_mem_mib[i]) for i in mem) > prof.mem_capacity_mib:
                continue
            grpT[S] = min(_group_T(prof, mem, lv) for lv in range(3))
        INF = float("inf")
        best = {(0, 0): 0.0}
        # dp over (covered set, #groups): min of max group T; groups contain lowest uncovered
        dp = {0: {0: 0.0}}
        for S in range(0, full + 1):
            if S not in dp:
                continue
            low = next((i for i in range(n) if not S >> i & 1), None)
            if low is None:
                continue
            rest = full & ~S & ~(1 << low)
            sub = rest
            while True:
                B = sub | (1 << low)
                if B in grpT:
                    for k, v in dp[S].items():
                        if k + 1 <= g:
                            nv = max(v, grpT[B])
                            dd = dp.setdefault(S | B, {})
                            if nv < dd.get(k + 1, INF):
                                dd[k + 1] = nv
                if sub == 0:
                    break
                sub = (sub - 1) & rest
        minT = min(dp[full].values())
        assert r["best"][0][2] == pytest.approx(minT, rel=1e-12)
        assert r["best"][0][1] == pytest.approx(r["tseq"] / minT, rel=1e-12)


def test_score_window_equals_per_index_scoring():
    """oracle.score_window (every configuration of a window, enumeration
    order) == oracle.config + oracle.score index by index (the extraction
    path), NaN exactly where infeasible."""
    import math
    import oracle
    from synth import make_profile, Query, PER_GPU, PER_CLIENT
    for scope, arch in ((PER_GPU, [11, 2, 0, 12, 5, 1, 3]), (PER_CLIENT, None)):
        prof = make_profile(7 if arch else 6, levels=(25, 50, 75, 100), seed=41, archetypes=arch)
        q = Query(prof.n_workflows, 3, 4, (50, 100), scope, ((1, 1),), False)
        lo, hi = 37, 37 + 700
        T, E = oracle.score_window(prof, q.with_range(lo, hi))
        for i in range(lo, hi):
            ok, t, e = oracle.score(prof, q, *oracle.config(q, i))
            if ok:
                assert (T[i - lo], E[i - lo]) == (t, e)
            else:
                assert math.isnan(T[i - lo]) and math.isnan(E[i - lo])
