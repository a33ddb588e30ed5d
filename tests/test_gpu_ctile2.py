"""GPU parity of the group-table PER_CLIENT tile kernel (kernel_path 6,
search_ctile2.cuh): PER_CLIENT, 4 levels per client, groups of <= 4 clients
-- the literal per-client reading (BASELINE.json north star "per-client
active-thread percentage") at c3 scale ("c3-client", SURVEY
8(d): 12 workflows, 8 GPUs, <= 4 clients per GPU, 5.5e13 configurations).
Full small spaces, ragged windows, unit-splitting chunk sizes, shards, the
c3-client windows, every weight-count template (1, 2, 4, 8), bitwise against
the oracle (test_gpu_parity.check) and against the older per-client tile
kernel (path 5)."""
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, Query, PER_CLIENT
from test_gpu_parity import check, _windows

pytestmark = pytest.mark.gpu

LV = (25, 50, 75, 100)
SWEEP = ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1))


def c3client():
    prof, q = config("c3")
    return prof, Query(12, 8, 4, LV, PER_CLIENT, ((1, 1),), True)


@pytest.mark.parametrize("n,g,c,ws,pareto,seed", [
    (6, 3, 3, ((1, 1),), True, 1), (7, 4, 2, SWEEP, True, 2), (7, 3, 4, ((1, 0), (0, 1)), False, 3),
    (8, 4, 4, (), True, 4), (6, 6, 1, ((2, 1), (1, 1)), True, 5), (8, 8, 3, ((1, 1), (2, 1), (1, 0), (0, 1)), True, 6),
])
def test_ctile2_small_full_and_windows(n, g, c, ws, pareto, seed):
    prof = make_profile(n, levels=LV, seed=600 + seed)
    q = Query(n, g, c, LV, PER_CLIENT, ws, pareto)
    sch = S.Scheduler(prof)
    res = sch.search(q)
    assert res.stats["kernel_path"] == 6
    check(res, oracle.search(prof, q), q)
    tot = S.count(q)
    rnd = random.Random(seed)
    for _ in range(3):
        lo = rnd.randrange(tot)
        qw = q.with_range(lo, min(tot, lo + rnd.randint(1, 60_000)))
        r2 = sch.search(qw)
        assert r2.stats["kernel_path"] == 6
        check(r2, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("cl", [12, 14, 16])
def test_ctile2_small_chunks_and_shards(cl):
    """Units smaller than a partition (4^9 configurations): tiles straddle unit
    boundaries; shards of small chunks merged equal the one-shot search."""
    prof = make_profile(9, levels=LV, seed=640)
    q = Query(9, 4, 3, LV, PER_CLIENT, ((1, 1), (2, 1)), True)
    sch = S.Scheduler(prof)
    one = sch.search(q, chunk_log2=cl)
    assert one.stats["kernel_path"] == 6
    check(one, oracle.search_parallel(prof, q), q)
    parts = [sch.search(q, shard=(r, 3), chunk_log2=cl) for r in range(3)]
    mb, mp = S.merge([x.best for x in parts], [x.pareto for x in parts], 2)
    assert [(b.index, b.score64) for b in mb] == [(b.index, b.score64) for b in one.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in mp] == \
        [(p.index, p.makespan_s, p.energy_j) for p in one.pareto]
    assert sum(x.stats["n_configs"] for x in parts) == S.count(q)


def test_ctile2_c3client_windows():
    prof, q = c3client()
    tot = S.count(q)
    assert tot == 55_045_542_379_520
    sch = S.Scheduler(prof)
    rnd = random.Random(77)
    for lo, hi in _windows(tot, 1 << 24, rnd, 300_000) + [((5 << 24) + 12345, (5 << 24) + 12345 + 400_000)]:
        qw = q.with_range(lo, hi)
        res = sch.search(qw)
        assert res.stats["kernel_path"] == 6
        check(res, oracle.search(prof, qw), qw)


def test_ctile2_equals_path5_on_a_c3client_slice(monkeypatch):
    """A 2^30-configuration stretch of c3-client (64 whole partitions) on the
    group-table kernel equals the per-client tile kernel (path 5) bitwise,
    and its picks re-score bitwise in the oracle."""
    prof, q = c3client()
    lo = 5000 << 24   # 64 feasible partitions (partitions 1000..1063 are all memory-infeasible)
    qw = q.with_range(lo, lo + (1 << 30))
    sch = S.Scheduler(prof)
    r6 = sch.search(qw)
    assert r6.stats["kernel_path"] == 6
    monkeypatch.setenv("SCHED_KERNEL", "ctile")
    r5 = sch.search(qw)
    assert r5.stats["kernel_path"] == 5
    assert [(b.index, b.score64) for b in r6.best] == [(b.index, b.score64) for b in r5.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in r6.pareto] == \
        [(p.index, p.makespan_s, p.energy_j) for p in r5.pareto]
    assert r6.stats["n_configs"] == r5.stats["n_configs"] == 1 << 30
    assert r6.stats["n_feasible"] > 0 and all(b.valid for b in r6.best)
    for p in list(r6.pareto) + list(r6.best):
        ok, T, E = oracle.score(prof, q, *oracle.config(q, p.index))
        assert ok and (T, E) == (p.makespan_s, p.energy_j)
