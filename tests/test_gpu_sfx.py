"""GPU parity of the L = 1 suffix kernel (kernel_path 3, search_sfx.cuh)
against the CPU oracle: full spaces, ragged windows, small chunks (unit and
prefix boundaries inside every chunk) and shards, capped and uncapped
client counts, every weight set shape (none = Pareto only, the c5 sweep).
The bar is that of test_gpu_parity.check: indices, fp64 scores and the
Pareto set bitwise equal, counts exact, fp32 scores within 1e-5."""
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, Query, PER_GPU
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

SWEEP = ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1))


@pytest.fixture
def sfx(monkeypatch):
    monkeypatch.setenv("SCHED_KERNEL", "sfx")


CASES = [
    # n, g, c, weights, seed         (n < 8: suffix length 4, else 6)
    (6, 3, 3, ((1, 1),), 1),
    (7, 4, 2, SWEEP, 2),
    (8, 4, 3, SWEEP, 3),
    (9, 8, 9, ((1, 1), (2, 1)), 4),      # uncapped
    (10, 5, 3, (), 5),                   # Pareto only
    (10, 8, 2, ((1, 0), (0, 1)), 6),
    (11, 4, 4, ((2, 1),), 7),
    (12, 6, 3, SWEEP, 8),
    (9, 3, 4, ((1, 2), (4, 4)), 9),
    (8, 8, 1, ((1, 1),), 10),            # singletons only
]


@pytest.mark.parametrize("n,g,c,ws,seed", CASES)
def test_sfx_full_and_windows(sfx, n, g, c, ws, seed):
    prof = make_profile(n, levels=(100,), seed=seed, g=g, c=c)
    q = Query(n, g, c, (100,), PER_GPU, ws, True)
    sch = S.Scheduler(prof)
    res = sch.search(q)
    assert res.stats["kernel_path"] == 3
    check(res, oracle.search(prof, q), q)
    tot = S.count(q)
    rnd = random.Random(seed)
    for _ in range(3):
        lo = rnd.randrange(tot)
        hi = min(tot, lo + rnd.randint(1, 50_000))
        qw = q.with_range(lo, hi)
        r2 = sch.search(qw)
        assert r2.stats["kernel_path"] == 3
        check(r2, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("n,g,c,ws,seed", [(10, 5, 3, SWEEP, 21), (11, 8, 3, ((1, 1),), 22)])
def test_sfx_small_chunks_and_shards(sfx, n, g, c, ws, seed):
    """chunk_log2 = 12: every 4096-index chunk cuts prefixes; R shards merged
    must equal the single search and the oracle."""
    prof = make_profile(n, levels=(100,), seed=seed, g=g, c=c)
    q = Query(n, g, c, (100,), PER_GPU, ws, True)
    sch = S.Scheduler(prof)
    one = sch.search(q, chunk_log2=12)
    ref = oracle.search(prof, q)
    check(one, ref, q)
    for R in (2, 3):
        bests, pars, ncfg = [], [], 0
        for r in range(R):
            res = sch.search(q, shard=(r, R), chunk_log2=12)
            bests.append(res.best)
            pars.append(res.pareto)
            ncfg += res.stats["n_configs"]
        mb, mp = S.merge(bests, pars, len(ws))
        assert ncfg == S.count(q)
        assert [(b.index, b.score64) for b in mb] == [(b.index, b.score64) for b in one.best]
        assert [(p.index, p.makespan_s, p.energy_j) for p in mp] == \
            [(p.index, p.makespan_s, p.energy_j) for p in one.pareto]


def test_sfx_c5_windows(sfx):
    """c5 (20 workflows, 8 GPUs, <= 3 clients, the 7-weight sweep) windows."""
    prof, q = config("c5")
    tot = S.count(q)
    sch = S.Scheduler(prof)
    rnd = random.Random(17)
    wins = [(0, 200_000), (tot - 200_000, tot), ((1 << 24) - 100_000, (1 << 24) + 100_000)]
    wins += [(x, x + 200_000) for x in (rnd.randrange(tot - 200_000) for _ in range(4))]
    for lo, hi in wins:
        qw = q.with_range(lo, hi)
        res = sch.search(qw)
        assert res.stats["kernel_path"] == 3
        check(res, oracle.search(prof, qw), qw)


def test_sfx_equals_pair_kernel(monkeypatch):
    """Same window of c5 on the suffix kernel and on the pair kernel."""
    prof, q = config("c5")
    qw = q.with_range(123_456_789_012, 123_456_789_012 + (1 << 23))
    sch = S.Scheduler(prof)
    monkeypatch.setenv("SCHED_KERNEL", "sfx")
    a = sch.search(qw)
    monkeypatch.setenv("SCHED_KERNEL", "dfs")
    b = sch.search(qw)
    assert a.stats["kernel_path"] == 3 and b.stats["kernel_path"] == 2
    assert a.stats["n_configs"] == b.stats["n_configs"] == 1 << 23
    assert a.stats["n_feasible"] == b.stats["n_feasible"]
    assert [(x.index, x.score64) for x in a.best] == [(x.index, x.score64) for x in b.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in a.pareto] == \
        [(p.index, p.makespan_s, p.energy_j) for p in b.pareto]
