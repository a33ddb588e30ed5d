"""Pins of the oracle's scoring-model variants (DESIGN.md
readings R26 COUNT_IDLE, R27 NO_INTERFERENCE, R28 POWER_CAP) against brute
force (O2, independent enumeration and transcription), limits that reduce
to the canonical model, closed forms in exact rational arithmetic on the
paper's Table II / III numbers, and an exact-rational feasibility count.
Each test names the mistake it would catch."""
import itertools
from fractions import Fraction

import numpy as np
import pytest

import oracle
import oracle.brute as br
from synth import make_profile, table_iii_combo1, Query, PER_CLIENT, PER_GPU

COUNT_IDLE, NO_INTERFERENCE, POWER_CAP = 1, 2, 4
W = ((1, 0), (0, 1), (1, 1), (2, 1), (1, 3))


def _fr(x):
    return Fraction(float(np.float32(x)))


def _same(r1, r2):
    assert [b[:4] if b else None for b in r1["best"]] == [b for b in r2["best"]]
    assert r1["pareto"] == r2["pareto"]
    assert r1["nfeasible"] == r2["nfeasible"] and r1["nconfigs"] == r2["nconfigs"]
    assert r1["tseq"] == r2["tseq"] and r1["eseq"] == r2["eseq"]


@pytest.mark.parametrize("model", [1, 2, 4, 3, 5, 6, 7])
@pytest.mark.parametrize("seed", range(4))
def test_variants_o1_equals_o2(model, seed):
    """O1 (enum.c) == O2 (brute.py) bitwise for every variant combination.
    Catches: a variant applied in a different order or to the wrong term
    on one side (e.g. cap before the stretch, idle energy per group)."""
    n = 5
    prof = make_profile(n, levels=(25, 50, 100), seed=100 + seed)
    q = Query(n, 3, 3 + seed % 3, (50, 100), seed % 2, W, True, model=model, power_cap=130.0)
    _same(oracle.search(prof, q), br.search(prof, q))


def test_power_cap_unbounded_is_canonical():
    """P_cap far above every group's power: identical (bitwise) to the
    canonical model.  Catches: the cap changing uncapped groups or the
    sequential energy formula (p*t kept for uncapped tasks)."""
    for seed in range(3):
        prof = make_profile(6, levels=(50, 100), seed=seed)
        q0 = Query(6, 3, 6, (50, 100), PER_GPU, W, True)
        q4 = Query(6, 3, 6, (50, 100), PER_GPU, W, True, model=POWER_CAP, power_cap=1e7)
        _same(oracle.search(prof, q0), oracle.search(prof, q4))


def test_power_cap_closed_form_combo1():
    """Table III combo 1 (Table II), P_cap = 200 W:
    LAMMPS 4x alone draws 258.38 W > 200 W, so it runs t' = t (p - P_s) /
    (P_cap - P_s) and spends exactly P_cap * t'; AthenaPK (88.86 W) is not
    capped.  Together, D = sum dyn over T: the group is capped iff
    D / (P_cap - P_s) > T.  Exact rationals.  Catches: wrong capped time
    (e.g. t * p / P_cap, which does not conserve dynamic energy)."""
    prof = table_iii_combo1((0.05, 0.10))
    tA, tL = _fr(prof.solo_time_s[0, 0]), _fr(prof.solo_time_s[1, 0])
    pA, pL = _fr(prof.solo_power_w[0, 0]), _fr(prof.solo_power_w[1, 0])
    Ps, Pc = Fraction(60), Fraction(200)
    tL2 = tL * (pL - Ps) / (Pc - Ps)
    assert tL2 > tL
    q = Query(2, 2, 2, (100,), PER_GPU, ((1, 0),), True, model=POWER_CAP, power_cap=200.0)
    ts, es = oracle.constants(prof, q)
    assert ts == pytest.approx(float(max(tA, tL2)), rel=1e-14)
    assert es == pytest.approx(float(pA * tA + Pc * tL2), rel=1e-14)
    # together on one GPU
    uA, uL, bA, bL = (_fr(prof.sm_util[0, 0]), _fr(prof.sm_util[1, 0]),
                      _fr(prof.bw_util[0, 0]), _fr(prof.bw_util[1, 0]))
    cg = max(Fraction(1), uA + uL, bA + bL)
    T = max(tA * (1 + _fr(0.05)) * cg, tL * (1 + _fr(0.10)) * cg)
    D = (pA - Ps) * tA + (pL - Ps) * tL
    T2 = max(T, D / (Pc - Ps))
    ok, To, Eo = oracle.score(prof, q, [0, 0], [0])
    assert ok and To == pytest.approx(float(T2), rel=1e-14)
    assert Eo == pytest.approx(float(Ps * T2 + D), rel=1e-14)


def test_count_idle_closed_form_combo1():
    """COUNT_IDLE on combo 1 with G = 2: E = G P_s T + sum dyn and E_seq =
    G P_s T_seq + sum dyn (every GPU powered for the whole makespan).
    Exact rationals on the paper's numbers.  Catches: idle energy counted
    only for unused GPUs, or missing from the baseline."""
    prof = table_iii_combo1((0.05, 0.10))
    tA, tL = _fr(prof.solo_time_s[0, 0]), _fr(prof.solo_time_s[1, 0])
    pA, pL = _fr(prof.solo_power_w[0, 0]), _fr(prof.solo_power_w[1, 0])
    uA, uL, bA, bL = (_fr(prof.sm_util[0, 0]), _fr(prof.sm_util[1, 0]),
                      _fr(prof.bw_util[0, 0]), _fr(prof.bw_util[1, 0]))
    Ps = Fraction(60)
    D = (pA - Ps) * tA + (pL - Ps) * tL
    q = Query(2, 2, 2, (100,), PER_GPU, ((1, 0), (0, 1)), True, model=COUNT_IDLE)
    ts, es = oracle.constants(prof, q)
    assert ts == pytest.approx(float(max(tA, tL)), rel=1e-15)
    assert es == pytest.approx(float(2 * Ps * max(tA, tL) + D), rel=1e-14)
    cg = max(Fraction(1), uA + uL, bA + bL)
    T = max(tA * (1 + _fr(0.05)) * cg, tL * (1 + _fr(0.10)) * cg)
    ok, To, Eo = oracle.score(prof, q, [0, 0], [0])
    assert ok and Eo == pytest.approx(float(2 * Ps * T + D), rel=1e-14)
    ok, To, Eo = oracle.score(prof, q, [0, 1], [0, 0])   # separate GPUs = the sequential schedule
    assert ok and Eo == es and To == ts


def test_count_idle_singletons_are_sequential():
    """N <= G, every workflow alone at 100 %: X = Y = 1 under COUNT_IDLE too.
    Catches: G vs k (used GPUs) in the idle term."""
    for seed in range(4):
        n = 4
        prof = make_profile(n, levels=(50, 100), seed=seed)
        q = Query(n, n + 2, n, (50, 100), PER_GPU, W, True, model=COUNT_IDLE)
        ts, es = oracle.constants(prof, q)
        ok, T, E = oracle.score(prof, q, list(range(n)), [1] * n)
        assert ok and ts / T == 1.0 and es / E == pytest.approx(1.0, abs=1e-15)


def test_no_interference_feasible_count_exact():
    """NO_INTERFERENCE feasibility decided in exact rationals of the fp32
    inputs (memory <= cap, and per group sum u <= 1 and sum bw <= 1) must
    match the oracle's feasible count (PAPER.md L87 predicate).  Catches:
    >= vs >, a predicate on one resource only, or on the wrong level."""
    for seed in range(4):
        n = 5
        prof = make_profile(n, levels=(50, 100), seed=200 + seed)
        q = Query(n, 3, 3, (50, 100), PER_CLIENT, (), True, model=NO_INTERFERENCE)
        sp = br.space(n, 3, 3, 2, PER_CLIENT)
        pct = [int(x) for x in prof.level_pct]
        lev = [pct.index(50), pct.index(100)]
        cnt = 0
        for rgs, dig in sp:
            ok = True
            for g in range(max(rgs) + 1):
                mem = [i for i in range(n) if rgs[i] == g]
                if sum(int(prof.max_mem_mib[i]) for i in mem) > int(prof.mem_capacity_mib):
                    ok = False
                if sum(_fr(prof.sm_util[i, lev[dig[i]]]) for i in mem) > 1:
                    ok = False
                if sum(_fr(prof.bw_util[i, lev[dig[i]]]) for i in mem) > 1:
                    ok = False
            cnt += ok
        r = oracle.search(prof, q)
        assert r["nfeasible"] == cnt
        assert r["nconfigs"] == len(sp)
