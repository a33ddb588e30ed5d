"""Pins of the oracle's TIME_SLICE variant (SURVEY 8(f) N4 "time-slicing
model"; reading R30: without MPS the clients of
a GPU take turns on the whole device, so a group's makespan is the sum of
its members' solo times and there is no contention or co-run slowdown).

Pinned against O2 (independent enumeration and transcription), invariances
the reading implies, a textbook reduction (the throughput optimum is the
minimum-makespan assignment of the solo times to <= G machines, computed
here by an independent brute force in exact rationals) and the exact
single-GPU identities X = 1, Y = 1.  Each test names the mistake it catches."""
import copy
import itertools
from fractions import Fraction

import numpy as np
import pytest

import oracle
import oracle.brute as br
from synth import make_profile, Query, PER_CLIENT, PER_GPU

COUNT_IDLE, POWER_CAP, TIME_SLICE = 1, 4, 8
W = ((1, 0), (0, 1), (1, 1), (2, 1))


def _same(r1, r2):
    assert [b[:4] if b else None for b in r1["best"]] == [b for b in r2["best"]]
    assert r1["pareto"] == r2["pareto"]
    assert r1["nfeasible"] == r2["nfeasible"] and r1["nconfigs"] == r2["nconfigs"]
    assert r1["tseq"] == r2["tseq"] and r1["eseq"] == r2["eseq"]


@pytest.mark.parametrize("model", [8, 9, 12, 13])
@pytest.mark.parametrize("seed", range(4))
def test_time_slice_o1_equals_o2(model, seed):
    """O1 (enum.c) == O2 (brute.py) bitwise, alone and with COUNT_IDLE /
    POWER_CAP.  Catches: the group cap applied on top of the per-slice cap,
    a max instead of the sum, the stretch c_g left in on one side."""
    n = 5
    prof = make_profile(n, levels=(25, 50, 100), seed=700 + seed)
    q = Query(n, 3, 3 + seed % 3, (50, 100), seed % 2, W, True, model=model, power_cap=130.0)
    _same(oracle.search(prof, q), br.search(prof, q))


@pytest.mark.parametrize("seed", range(3))
def test_time_slice_ignores_corun_and_utilisation(seed):
    """R30: no concurrency -> the co-run matrix and the SM / BW utilisations
    cannot matter.  Redrawing them leaves every result bitwise unchanged.
    Catches: sigma or c_g still applied under time slicing."""
    n = 6
    prof = make_profile(n, levels=(50, 100), seed=seed)
    q = Query(n, 3, 6, (50, 100), PER_GPU, W, True, model=TIME_SLICE)
    alt = copy.deepcopy(prof)
    rng = np.random.default_rng(seed)
    alt.corun_slowdown[...] = rng.uniform(0.0, 3.0, alt.corun_slowdown.shape).astype(np.float32)
    alt.sm_util[...] = rng.uniform(0.5, 1.0, alt.sm_util.shape).astype(np.float32)
    alt.bw_util[...] = rng.uniform(0.5, 1.0, alt.bw_util.shape).astype(np.float32)
    _same(oracle.search(prof, q), oracle.search(alt, q))
    # and the canonical model does see them (the redraw is not a no-op)
    q0 = Query(n, 3, 6, (50, 100), PER_GPU, W, True)
    assert oracle.search(prof, q0)["best"] != oracle.search(alt, q0)["best"]


def _min_makespan(prof, n, g, c, levels):
    """Independent brute force in exact rationals: every labeling of the n
    workflows onto g machines (<= c per machine, memory within capacity) and
    every per-client level choice; makespan = max over machines of the sum
    of the float32 solo times (classic P||Cmax)."""
    pct = [int(x) for x in prof.level_pct]
    li = [pct.index(v) for v in levels]
    t = [[Fraction(float(prof.solo_time_s[i, l])) for l in li] for i in range(n)]
    mem = [int(prof.max_mem_mib[i]) for i in range(n)]
    best = None
    for lab in itertools.product(range(g), repeat=n):
        ok = all(lab.count(m) <= c and sum(mem[i] for i in range(n) if lab[i] == m) <= int(prof.mem_capacity_mib)
                 for m in range(g))
        if not ok:
            continue
        # the best level of a client is its fastest one (each term independent)
        loads = [sum((min(t[i]) for i in range(n) if lab[i] == m), Fraction(0)) for m in range(g)]
        ms = max(loads)
        best = ms if best is None or ms < best else best
    return best


@pytest.mark.parametrize("seed", range(4))
def test_time_slice_throughput_is_min_makespan(seed):
    """Throughput optimum under time slicing = the minimum makespan of the
    solo times on <= G machines (textbook P||Cmax), PER_CLIENT levels.
    Catches: a dropped member, a wrong group's time summed, levels ignored."""
    n, g = 6, 3
    prof = make_profile(n, levels=(50, 100), seed=40 + seed, g=g, c=4)
    q = Query(n, g, 4, (50, 100), PER_CLIENT, ((1, 0),), False, model=TIME_SLICE)
    r = oracle.search(prof, q)
    T = r["best"][0][2]
    ref = _min_makespan(prof, n, g, 4, (50, 100))
    assert abs(Fraction(T) - ref) <= ref * Fraction(1, 2 ** 50)


@pytest.mark.parametrize("seed", range(4))
def test_time_slice_single_gpu_is_sequential(seed):
    """G = 1: the only partition is one group; at the 100 % level its time-
    sliced makespan is the sequential list schedule summed in the same queue
    order (X == 1 bitwise), and its energy P_s*sum t + sum (p - P_s) t is
    sum p t = E_seq in exact arithmetic (Y == 1 to rounding).  With the cap
    every slice is throttled exactly as the baseline's solo task.
    Catches: a stretch / co-run term, the group cap instead of per slice."""
    n = 4
    prof = make_profile(n, levels=(50, 100), seed=seed)
    for model, cap in ((TIME_SLICE, 0.0), (TIME_SLICE | POWER_CAP, 120.0)):
        q = Query(n, 1, n, (100,), PER_GPU, ((1, 0), (0, 1)), True, model=model, power_cap=cap)
        r = oracle.search(prof, q)
        (i0, fx, T, E), (i1, fy, T1, E1) = r["best"]
        assert i0 == 0 and i1 == 0
        assert T == r["tseq"] and fx == 1.0
        assert abs(E / r["eseq"] - 1.0) < 1e-14
