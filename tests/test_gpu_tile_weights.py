"""The PER_GPU tile kernel (kernel_path 1, the c3 / c4 path) with any
product-metric set ("[throughput x efficiency] or [throughput
x throughput x efficiency]", L178 "different product metrics"): weight sets
without a compiled-in specialisation run the run-time-exponent variant
(WS_RT).  c4-size windows (start, end, chunk boundaries, random) and small
full spaces, bitwise against the oracle (test_gpu_parity.check)."""
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, Query, PER_GPU
from test_gpu_parity import check, _windows

pytestmark = pytest.mark.gpu

SETS = {
    "c1_set": ((1, 0), (0, 1), (1, 1), (2, 1)),                       # BASELINE configs[0]'s objectives
    "c5_sweep": ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1)),   # configs[4]'s sweep
    "eight": ((1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (4, 4)),
    "single_12": ((1, 2),),                                            # WS_RT4N (no b = 0 weight)
    "rt4n": ((1, 1), (2, 1), (1, 2)),                                  # WS_RT4N
    "rtn6": ((1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (2, 2)),          # WS_RTN (5..8 weights, every b >= 1)
}


@pytest.mark.parametrize("name", list(SETS))
def test_runtime_weights_c4_windows(name):
    prof, q = config("c4")
    qn = Query(q.n, q.g, q.c, q.levels, q.scope, SETS[name], True)
    tot = S.count(qn)
    sch = S.Scheduler(prof)
    rnd = random.Random(len(name))
    for lo, hi in _windows(tot, 1 << 24, rnd, 300_000):
        qw = qn.with_range(lo, hi)
        res = sch.search(qw)
        assert res.stats["kernel_path"] == 1
        check(res, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("seed", range(4))
def test_runtime_weights_small_full(seed):
    rnd = random.Random(seed)
    n, g = rnd.randint(6, 9), rnd.randint(5, 8)
    ws = tuple(rnd.sample([(1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (4, 4)], rnd.randint(3, 8)))
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=300 + seed)
    q = Query(n, g, n, (25, 50, 75, 100), PER_GPU, ws, seed % 2 == 0)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 1
    check(res, oracle.search(prof, q), q)


@pytest.mark.parametrize("levels", [(50, 100), (50, 75, 100), (25, 75, 100)])
@pytest.mark.parametrize("ws", [(), ((1, 1),), ((1, 0), (0, 1), (1, 1), (2, 1)), ((1, 2), (3, 1))])
def test_two_and_three_levels_c4_windows(levels, ws):
    """PER_GPU with 2 or 3 searched MPS levels (P:L75 granularity) on the tile
    kernel's per-configuration path (kernel_path 1: k_tile only
    took L = 4): c4-size windows bitwise against the oracle."""
    prof, q = config("c4")
    qn = Query(q.n, q.g, q.c, levels, q.scope, ws, True)
    tot = S.count(qn)
    sch = S.Scheduler(prof)
    rnd = random.Random(len(levels) * 10 + len(ws))
    for lo, hi in _windows(tot, 1 << 24, rnd, 200_000):
        qw = qn.with_range(max(0, lo), min(tot, hi))
        res = sch.search(qw)
        assert res.stats["kernel_path"] == 1
        check(res, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("seed", range(4))
def test_two_and_three_levels_small_full(seed):
    rnd = random.Random(100 + seed)
    n, g = rnd.randint(5, 9), rnd.randint(2, 8)
    levels = rnd.choice(((50, 100), (25, 50, 100), (75, 100), (25, 50, 75)))
    ws = tuple(rnd.sample([(1, 0), (0, 1), (1, 1), (2, 1), (1, 2)], rnd.randint(0, 4)))
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=400 + seed)
    q = Query(n, g, rnd.randint(max(1, -(-n // g)), n), levels, PER_GPU, ws, True,
              model=4 if seed == 3 else 0, power_cap=170.0)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 1
    check(res, oracle.search(prof, q), q)
