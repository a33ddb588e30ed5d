"""GPU parity: the CUDA search (through the C ABI) against the CPU oracle.

Bar (BASELINE.json north_star): configuration counts, chosen indices (ties
-> lowest index) and the Pareto set bit-exact; the fp64 scores of the picks
bitwise equal to the oracle's; the fp32 hot-loop scores within 1e-5
relative of the oracle's fp64.
"""
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import CONFIGS, config, make_profile, Query, PER_CLIENT, PER_GPU

pytestmark = pytest.mark.gpu

REL32 = 1e-5


def check(res, ref, q, sched=None):
    nw = len(q.weights)
    for w in range(nw):
        r = ref["best"][w]
        b = res.best[w]
        if r is None:
            assert not b.valid
            continue
        assert b.valid
        assert b.index == r[0], (w, b.index, r)
        assert b.score64 == r[1] and b.makespan_s == r[2] and b.energy_j == r[3]
        assert abs(b.score32 / r[1] - 1) <= REL32
        assert abs(b.x32 / (ref["tseq"] / r[2]) - 1) <= REL32
        assert abs(b.y32 / (ref["eseq"] / r[3]) - 1) <= REL32
    if q.want_pareto:
        got = [(p.index, p.makespan_s, p.energy_j) for p in res.pareto]
        assert got == ref["pareto"]
        for p in res.pareto:
            assert abs(p.x32 / (ref["tseq"] / p.makespan_s) - 1) <= REL32
            assert abs(p.y32 / (ref["eseq"] / p.energy_j) - 1) <= REL32
    assert res.stats["n_configs"] == ref["nconfigs"]
    assert res.stats["n_feasible"] == ref["nfeasible"]


def _cases():
    rnd = random.Random(2024)
    out = []
    for t in range(40):
        n = rnd.randint(2, 8)
        g = rnd.randint(1, 5)
        c = rnd.randint(max(1, -(-n // g)), n)
        L = rnd.randint(1, 4)
        levels = tuple(sorted(rnd.sample([25, 50, 75, 100], L)))
        scope = rnd.choice([PER_CLIENT, PER_GPU])
        if scope == PER_CLIENT and L ** n > 5000:
            scope = PER_GPU
        ws = tuple(rnd.sample([(1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (4, 4)],
                              rnd.randint(0, 5)))
        out.append((t, n, g, c, levels, scope, ws))
    return out


@pytest.mark.parametrize("t,n,g,c,levels,scope,ws", _cases())
def test_small_spaces_full(t, n, g, c, levels, scope, ws):
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=500 + t)
    q = Query(n, g, c, levels, scope, ws, True)
    ref = oracle.search(prof, q)
    res = S.Scheduler(prof).search(q)
    check(res, ref, q)


def test_c1_full():
    prof, q = config("c1")
    check(S.Scheduler(prof).search(q), oracle.search(prof, q), q)


def test_c2_full():
    prof, q = config("c2")
    q2 = Query(q.n, q.g, q.c, q.levels, q.scope, ((1, 0), (1, 1), (0, 1)), True)
    ref = oracle.search_parallel(prof, q2)
    check(S.Scheduler(prof).search(q2), ref, q2)


def _windows(tot, chunk, rnd, size):
    ws = [(0, size), (tot - size, tot), (chunk - size // 2, chunk + size // 2),
          (3 * chunk - 7, 3 * chunk + size - 7)]
    ws += [(x, x + size) for x in (rnd.randrange(tot - size) for _ in range(4))]
    return ws


@pytest.mark.parametrize("name", ["c3", "c4", "c5"])
def test_windows_big_spaces(name):
    prof, q = config(name)
    tot = S.count(q)
    sch = S.Scheduler(prof)
    rnd = random.Random(11)
    for lo, hi in _windows(tot, 1 << 24, rnd, 300_000):
        qw = q.with_range(lo, hi)
        check(sch.search(qw), oracle.search(prof, qw), qw)


@pytest.mark.parametrize("R", [2, 3, 8])
def test_sharded_merge_equals_single(R):
    prof, q = config("c4")
    q = Query(q.n, q.g, q.c, q.levels, q.scope, ((1, 1), (2, 1), (1, 0)), True)
    lo = 123_456_789_000
    qw = q.with_range(lo, lo + 5 * (1 << 16) + 333)
    sch = S.Scheduler(prof)
    one = sch.search(qw, chunk_log2=16)
    bests, pars, ncfg = [], [], 0
    for r in range(R):
        res = sch.search(qw, shard=(r, R), chunk_log2=16)
        bests.append(res.best)
        pars.append(res.pareto)
        ncfg += res.stats["n_configs"]
    mb, mp = S.merge(bests, pars, 3)
    assert ncfg == one.stats["n_configs"] == qw.index_hi - qw.index_lo
    assert [b.index for b in mb] == [b.index for b in one.best]
    assert [b.score64 for b in mb] == [b.score64 for b in one.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in mp] == \
        [(p.index, p.makespan_s, p.energy_j) for p in one.pareto]
    check(one, oracle.search(prof, qw), qw)


def test_edge_cases():
    prof = make_profile(6, levels=(50, 100), seed=77)
    sch = S.Scheduler(prof)
    # empty window
    q = Query(6, 3, 6, (50, 100), PER_GPU, ((1, 1),), True, 10, 10)
    res = sch.search(q)
    assert res.stats["n_configs"] == 0 and res.status == S.sched.SCHED_E_INFEASIBLE
    # single configuration space: G = 1, one level
    q = Query(6, 1, 6, (100,), PER_GPU, ((1, 0), (0, 1)), True)
    check(sch.search(q), oracle.search(prof, q), q)
    # n = 1
    q = Query(1, 4, 1, (50, 100), PER_CLIENT, ((1, 1),), True)
    check(sch.search(q), oracle.search(prof, q), q)
    # all infeasible: two WarpX must share one GPU
    p2 = make_profile(3, levels=(100,), seed=1, archetypes=[11, 12, 11])
    q = Query(3, 1, 3, (100,), PER_GPU, ((1, 1),), True)
    res = S.Scheduler(p2).search(q)
    assert res.status == S.sched.SCHED_E_INFEASIBLE and not res.best[0].valid and res.pareto == []
    # ragged window inside a partition
    q = Query(6, 3, 6, (50, 100), PER_CLIENT, ((2, 1), (1, 2)), True, 37, 1001)
    check(sch.search(q), oracle.search(prof, q), q)


def test_c3_full_size_properties():
    """Full c3 (2.6e10 configs) in the bench launch configuration; the oracle
    checks the picks one by one and bounds them with random windows."""
    prof, q = config("c3")
    sch = S.Scheduler(prof)
    res = sch.search(q)
    tot = S.count(q)
    assert res.stats["n_configs"] == tot
    ts, es = oracle.constants(prof, q)
    b = res.best[0]
    ok, T, E = oracle.score(prof, q, *oracle.config(q, b.index))
    assert ok and b.makespan_s == T and b.energy_j == E
    assert b.score64 == oracle.objective(ts, es, T, E, 1, 1)
    for p in res.pareto:
        ok, T, E = oracle.score(prof, q, *oracle.config(q, p.index))
        assert ok and (T, E) == (p.makespan_s, p.energy_j)
    front = [(p.makespan_s, p.energy_j) for p in res.pareto]
    rnd = random.Random(5)
    for _ in range(6):
        lo = rnd.randrange(tot - 200_000)
        r = oracle.search(prof, q.with_range(lo, lo + 200_000))
        if r["best"][0] is not None:
            assert r["best"][0][1] < b.score64 or (r["best"][0][1] == b.score64 and r["best"][0][0] >= b.index)
        for _, T, E in r["pareto"]:
            assert any(t2 <= T and e2 <= E for t2, e2 in front)


def _certificate(name):
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", f"{name}_certificate.json")))
    front = [(float.fromhex(t), float.fromhex(e)) for t, e in g["front_T_E"]]
    best = [float.fromhex(b) for b in g["best_score64"]]
    return front, best


@pytest.mark.parametrize("name", ["c3", "c4", "c5"])
def test_full_space_vs_dp_certificate(name):
    """Full c3 / c4 / c5 search (c4: 2.07e14 configurations, ~60 s on one B200) in
    the bench's launch configuration vs the O3 subset-DP certificate
    (tests/golden/<cfg>_certificate.json, written by oracle/make_certificates.py):
    the Pareto front values and the optimum of every weight must be bitwise
    equal; every returned index is re-scored by the oracle."""
    prof, q = config(name)
    front, best = _certificate(name)
    res = S.Scheduler(prof).search(q)
    assert res.stats["n_configs"] == S.count(q)
    assert [(p.makespan_s, p.energy_j) for p in res.pareto] == front
    assert [b.score64 for b in res.best] == best
    for p in list(res.pareto) + list(res.best):
        ok, T, E = oracle.score(prof, q, *oracle.config(q, p.index))
        assert ok and (T, E) == (p.makespan_s, p.energy_j)


@pytest.mark.parametrize("n,g,c,ws,seed", [
    (9, 4, 3, ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1)), 1),
    (10, 5, 2, ((1, 1),), 2), (8, 8, 4, ((1, 1), (2, 1)), 3), (11, 4, 3, (), 4), (7, 3, 4, ((1, 0),), 5),
])
def test_partition_kernel_path(n, g, c, ws, seed, monkeypatch):
    """L = 1 spaces (every configuration is a partition) on the pair kernel
    (kernel_path 2, SCHED_KERNEL=dfs) must equal the oracle exactly."""
    monkeypatch.setenv("SCHED_KERNEL", "dfs")
    prof = make_profile(n, levels=(100,), seed=seed)
    q = Query(n, g, c, (100,), PER_GPU, ws, True)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 2
    check(res, oracle.search(prof, q), q)
    lo = S.count(q) // 3
    qw = q.with_range(lo, lo + 12345)
    res = S.Scheduler(prof).search(qw)
    check(res, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("n,g,c,ws,seed", [
    (8, 4, 8, ((1, 1),), 1), (9, 6, 3, ((1, 1), (2, 1)), 2), (7, 7, 7, (), 3), (9, 8, 9, ((1, 0),), 4),
])
def test_tile_kernel_path(n, g, c, ws, seed):
    """L = 4 PER_GPU spaces run on the tile kernel (kernel_path 1)."""
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, (25, 50, 75, 100), PER_GPU, ws, True)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 1
    check(res, oracle.search(prof, q), q)


def test_dense_local_front_window():
    """A 3.3e12-configuration c4 window in the middle of the space whose local
    Pareto front is dense inside the default staircase buckets (2^-7 relative
    T width): before the seed-pass re-bucketing it flooded the candidate
    buffer (SCHED_E_CAPACITY).  Must succeed, re-score exactly, and equal the
    merge of its two halves."""
    prof, q = config("c4")
    lo, n = 100_000_000_000_000, 3 << 40
    qw = q.with_range(lo, lo + n)
    sch = S.Scheduler(prof)
    res = sch.search(qw)
    assert res.status == S.sched.SCHED_OK and res.stats["n_configs"] == n
    assert res.stats["n_candidates"] < 1 << 20
    for p in list(res.pareto) + list(res.best):
        ok, T, E = oracle.score(prof, q, *oracle.config(q, p.index))
        assert ok and (T, E) == (p.makespan_s, p.energy_j)
    halves = [sch.search(q.with_range(lo, lo + n // 2)), sch.search(q.with_range(lo + n // 2, lo + n))]
    mb, mp = S.merge([h.best for h in halves], [h.pareto for h in halves], len(q.weights))
    assert [(b.index, b.score64) for b in mb] == [(b.index, b.score64) for b in res.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in mp] == \
        [(p.index, p.makespan_s, p.energy_j) for p in res.pareto]


@pytest.mark.parametrize("n,g,c,levels,scope", [
    (32, 2, 32, (100,), PER_GPU),          # maximum queue (SCHED_MAX_WORKFLOWS), 2^31 configurations
    (32, 16, 2, (100,), PER_GPU),          # maximum GPUs, pairs only: 32!/(2^16 16!) = 1.9e17
    (20, 16, 48, (50, 100), PER_GPU),      # maximum GPUs and MPS clients, no group table cap
    (13, 3, 13, (10, 20, 30, 40, 55, 70, 85, 100), PER_CLIENT),  # 8 searched levels (SCHED_MAX_SEARCH_LEVELS)
])
def test_maximum_sizes_windows(n, g, c, levels, scope):
    """Maximum sizes of the boundary (include/sched.h): windows at the start,
    the end and a ragged interior offset, bitwise against the oracle."""
    lv = tuple(sorted(set(levels)))
    # small-memory archetypes (Table II 1x rows) keep the large queues feasible
    arch = [(0, 3, 5, 9)[i % 4] for i in range(n)] if n >= 20 else None
    prof = make_profile(n, levels=lv, seed=900 + n + g, archetypes=arch)
    q = Query(n, g, c, lv, scope, ((1, 0), (1, 1), (0, 1)), True)
    tot = S.count(q)
    assert tot == oracle.count(q) and tot < 1 << 63
    sch = S.Scheduler(prof)
    for lo in (0, tot // 3 + 12345, tot - 150_000):
        qw = q.with_range(lo, min(tot, lo + 150_000))
        check(sch.search(qw), oracle.search(prof, qw), qw)


@pytest.mark.parametrize("n,g,c,ws,pareto,model,seed", [
    (6, 3, 3, ((1, 0), (0, 1), (1, 1), (2, 1)), True, 0, 11),
    (6, 2, 6, ((1, 1),), True, 4, 12),                 # POWER_CAP variant
    (7, 4, 7, ((1, 0),), False, 0, 13),
    (7, 4, 2, ((2, 1), (1, 3)), True, 0, 14),
    (6, 6, 6, (), True, 0, 15),                        # Pareto only, many groups
])
@pytest.mark.parametrize("kernel", ["ctile", "auto"])
def test_client_tile_kernel_path(n, g, c, ws, pareto, model, seed, kernel, monkeypatch):
    """PER_CLIENT, L = 4 spaces on the PER_CLIENT tile kernels (kernel_path 5;
    auto picks the group-table kernel, path 6, when groups have <= 4 clients):
    full space and ragged windows bitwise against the oracle."""
    if kernel != "auto":
        monkeypatch.setenv("SCHED_KERNEL", kernel)
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, (25, 50, 75, 100), PER_CLIENT, ws, pareto, model=model, power_cap=150.0)
    sch = S.Scheduler(prof)
    res = sch.search(q)
    assert res.stats["kernel_path"] == (5 if kernel == "ctile" or c > 4 else 6)
    check(res, oracle.search(prof, q), q)
    tot = S.count(q)
    for lo, hi in ((1000, 70_001), (tot // 2 - 4097, tot // 2 + 33_333), (tot - 50_000, tot)):
        qw = q.with_range(lo, hi)
        check(sch.search(qw), oracle.search(prof, qw), qw)


def test_bench_slice_launch_configuration():
    """One bench.py step exactly as it is timed (c4, shard (sigma, 64) of
    2^24-index chunks (bench.CHUNK_LOG2), 3.2e12 configurations): coverage equals the slice's
    index count, every returned configuration re-scores bitwise in the
    oracle, the slice's optimum never beats the O3 certificate's, and no
    sampled oracle window of the slice beats the slice's best or escapes its
    Pareto front."""
    import json
    import os
    prof, q = config("c4")
    import bench
    sigma, slices, cl = 5, 64, bench.CHUNK_LOG2
    tot = S.count(q)
    sch = S.Scheduler(prof)
    res = sch.search(q, shard=(sigma, slices), chunk_log2=cl)
    nch = (tot + (1 << cl) - 1) >> cl
    want = sum(min(tot, (c + 1) << cl) - (c << cl) for c in range(sigma, nch, slices))
    assert res.stats["n_configs"] == want
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c4_certificate.json")))
    for w, b in enumerate(res.best):
        assert b.valid and (b.index >> cl) % slices == sigma
        ok, T, E = oracle.score(prof, q, *oracle.config(q, b.index))
        assert ok and (T, E) == (b.makespan_s, b.energy_j)
        assert b.score64 <= float.fromhex(g["best_score64"][w])
    for p in res.pareto:
        assert (p.index >> cl) % slices == sigma
        ok, T, E = oracle.score(prof, q, *oracle.config(q, p.index))
        assert ok and (T, E) == (p.makespan_s, p.energy_j)
    front = [(p.makespan_s, p.energy_j) for p in res.pareto]
    rnd = random.Random(17)
    for _ in range(4):
        c = sigma + slices * rnd.randrange((nch - sigma) // slices - 1)  # whole chunks only
        lo = (c << cl) + rnd.randrange((1 << cl) - 200_000)
        r = oracle.search(prof, q.with_range(lo, lo + 200_000))
        for w, b in enumerate(res.best):
            x = r["best"][w]
            if x is not None:
                assert x[1] < b.score64 or (x[1] == b.score64 and x[0] >= b.index)
        for _, T, E in r["pareto"]:
            assert any(t2 <= T and e2 <= E for t2, e2 in front)
