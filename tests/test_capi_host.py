"""C-ABI library: loads, exports every symbol of include/sched.h, and its
host-side logic (count, unrank/rank, fp64 score, merge, validation) agrees
with the oracle.  No device compute (runs without a GPU)."""
import ctypes as C
import os
import random
import re

import numpy as np
import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from paper_conf_sc_weaverkmeh0m24_b200 import build as B
from synth import CONFIGS, config, make_profile, Query, PER_CLIENT, PER_GPU

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    B.build()


def test_exports_match_header():
    hdr = open(os.path.join(ROOT, "include", "sched.h")).read()
    decl = set(re.findall(r"^\s*(?:int|const char \*)\s*(sched_\w+)\s*\(", hdr, re.M))
    assert decl == set(S.EXPORTS)
    lib = C.CDLL(S.sched.SO_PATH)
    for name in decl:
        assert hasattr(lib, name), name


def test_so_is_sm100a():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {S.sched.SO_PATH}").read()
    assert "sm_100a" in out


@pytest.mark.parametrize("name", list(CONFIGS))
def test_count_unrank_rank_match_oracle(name):
    prof, q = config(name)
    tot = S.count(q)
    assert tot == oracle.count(q)
    rnd = random.Random(hash(name) & 0xffff)
    for idx in [0, 1, tot - 1, tot // 2] + [rnd.randrange(tot) for _ in range(40)]:
        a, lv = S.unrank(q, idx)
        oa, od = oracle.config(q, idx)
        assert a == oa
        assert lv == [od[i] if q.scope == PER_CLIENT else od[oa[i]] for i in range(q.n)]
        assert S.rank(q, a, lv) == idx


def test_unrank_bijection_small():
    for (n, g, c, L, sc) in [(5, 3, 2, 2, PER_GPU), (4, 2, 4, 2, PER_CLIENT), (6, 4, 3, 3, PER_GPU),
                             (7, 7, 7, 1, PER_GPU), (6, 2, 3, 2, PER_CLIENT)]:
        q = Query(n, g, c, tuple(range(L)), sc, ())
        tot = S.count(q)
        prev = None
        for idx in range(tot):
            a, lv = S.unrank(q, idx)
            assert S.rank(q, a, lv) == idx
            key = (tuple(a), tuple(lv[i] for i in range(n)) if sc == PER_CLIENT else
                   tuple(lv[a.index(b)] for b in range(max(a) + 1)))
            assert prev is None or key > prev      # strictly increasing (R4)
            prev = key


def test_count_too_large():
    q = Query(16, 8, 16, (0, 1, 2, 3), PER_CLIENT, ())
    with pytest.raises(S.SchedError) as e:
        S.count(q)
    assert e.value.status == S.sched.SCHED_E_TOO_LARGE


@pytest.mark.parametrize("name", ["c1", "c3", "c4", "c5"])
def test_host_score_bitwise_oracle(name):
    prof, q = config(name)
    sch = S.Scheduler(prof)
    tot = S.count(q)
    rnd = random.Random(5)
    ts, es = oracle.constants(prof, q)
    for idx in [0, tot - 1] + [rnd.randrange(tot) for _ in range(30)]:
        ok, T, E = oracle.score(prof, q, *oracle.config(q, idx))
        for w, (a, b) in enumerate(q.weights):
            p = sch.score(q, idx, w)
            assert p.valid == ok
            if ok:
                assert p.makespan_s == T and p.energy_j == E
                assert p.score64 == oracle.objective(ts, es, T, E, a, b)


@pytest.mark.parametrize("model", [1, 2, 4, 7, 8, 9, 12, 13])
@pytest.mark.parametrize("name", ["c2", "c4", "c5"])
def test_host_score_variants_bitwise_oracle(name, model):
    """Library fp64 host score (sched_score) under the scoring-model variants
    (R26-R28, R30) == the oracle's, bitwise, including the variant baselines."""
    import dataclasses
    prof, q = config(name)
    q = dataclasses.replace(q, model=model, power_cap=180.0)
    sch = S.Scheduler(prof)
    tot = S.count(q)
    rnd = random.Random(7)
    ts, es = oracle.constants(prof, q)
    nv = 0
    for idx in [0, tot - 1] + [rnd.randrange(tot) for _ in range(40)]:
        ok, T, E = oracle.score(prof, q, *oracle.config(q, idx))
        for w, (a, b) in enumerate(q.weights):
            p = sch.score(q, idx, w)
            assert p.valid == ok
            if ok:
                nv += 1
                assert p.makespan_s == T and p.energy_j == E
                assert p.score64 == oracle.objective(ts, es, T, E, a, b)
    assert nv > 0 or model & 2   # c5 groups of 3 mostly exceed 100 % SM


def test_variant_queries_validated():
    """POWER_CAP needs P_cap > P_s; unknown model bits and TIME_SLICE with
    NO_INTERFERENCE (R30) are rejected."""
    import dataclasses
    prof, q = config("c1")
    sch = S.Scheduler(prof)
    for bad in (dict(model=4, power_cap=50.0), dict(model=4, power_cap=0.0), dict(model=16),
                dict(model=10)):
        with pytest.raises(S.SchedError) as e:
            sch.score(dataclasses.replace(q, **bad), 0, 0)
        assert e.value.status == S.sched.SCHED_E_INVALID


def test_invalid_profiles_rejected():
    prof = make_profile(4, levels=(50, 100), seed=1)
    bad = make_profile(4, levels=(50, 100), seed=1)
    bad.solo_power_w[0, 0] = 10.0            # below static power
    with pytest.raises(S.SchedError):
        S.Scheduler(bad)
    bad = make_profile(4, levels=(50, 100), seed=1)
    bad.level_pct = np.array([25, 50], np.int32)   # no 100% column
    with pytest.raises(S.SchedError):
        S.Scheduler(bad)
    sch = S.Scheduler(prof)
    for q in [Query(5, 2, 4, (50, 100), PER_GPU, ()), Query(4, 0, 4, (50, 100), PER_GPU, ()),
              Query(4, 2, 4, (50, 100), PER_GPU, ((0, 0),)), Query(4, 2, 4, (50, 100), 3, ())]:
        with pytest.raises(S.SchedError):
            sch.workspace_size(q)


def test_merge_host():
    """sched_merge against a brute-force merge of random per-rank records."""
    rnd = random.Random(3)
    R, W = 4, 3
    rank_best, rank_par = [], []
    allpts = []
    for r in range(R):
        bl = []
        for w in range(W):
            p = S.Pick()
            p.valid = rnd.random() < 0.8
            p.index = rnd.randrange(1000)
            p.score64 = rnd.choice([1.0, 1.5, 2.0])
            bl.append(p)
        rank_best.append(bl)
        pl = []
        for _ in range(rnd.randrange(6)):
            p = S.Pick()
            p.valid = 1
            p.index = rnd.randrange(1000)
            p.makespan_s = rnd.choice([1.0, 2.0, 3.0])
            p.energy_j = rnd.choice([1.0, 2.0, 3.0])
            pl.append(p)
            allpts.append((p.makespan_s, p.energy_j, p.index))
        rank_par.append(pl)
    best, par = S.merge(rank_best, rank_par, W)
    for w in range(W):
        cands = [rank_best[r][w] for r in range(R) if rank_best[r][w].valid]
        if not cands:
            assert not best[w].valid
            continue
        exp = max(cands, key=lambda p: (p.score64, -p.index))
        assert (best[w].index, best[w].score64) == (exp.index, exp.score64)
    front = {}
    for t, e, i in allpts:
        if any((t2 <= t and e2 <= e and (t2 < t or e2 < e)) for t2, e2, _ in allpts):
            continue
        front[(t, e)] = min(i, front.get((t, e), i))
    exp = sorted([(t, e, i) for (t, e), i in front.items()])
    assert [(p.makespan_s, p.energy_j, p.index) for p in par] == exp


@pytest.mark.parametrize("seed", range(6))
def test_heuristic_rules_and_gap(seed):
    """The paper's rule-based scheduler: its configuration
    obeys criteria 2-4 where possible, round-trips through rank/unrank, is
    scored exactly like the oracle, and never beats the exhaustive optimum."""
    n, g = 7, 4
    prof = make_profile(n, levels=(50, 100), seed=60 + seed)
    q = Query(n, g, n, (50, 100), PER_GPU, ((1, 1), (1, 0), (0, 1)), True)
    sch = S.Scheduler(prof)
    ref = oracle.search(prof, q)
    for pr, lim in (("throughput", 2), ("energy", n)):
        try:
            a, lv, idx, pick = sch.heuristic(q, pr, 0)
        except S.SchedError as e:
            assert e.status == S.sched.SCHED_E_INFEASIBLE
            continue
        oa, od = oracle.config(q, idx)
        assert oa == a
        assert all(x == 1 for x in lv)                      # highest searched level (100 %)
        assert max(a.count(b) for b in set(a)) <= lim      # criterion 4
        for b in set(a):                                    # criterion 3
            assert sum(int(prof.max_mem_mib[i]) for i in range(n) if a[i] == b) <= prof.mem_capacity_mib
        ok, T, E = oracle.score(prof, q, oa, od)
        assert pick.valid == ok and pick.makespan_s == T and pick.energy_j == E
        assert pick.score64 <= ref["best"][0][1]


def test_binding_result_types_construct():
    """The binding's result containers build from plain values (the ctypes
    records stay plain Structures; SearchResult is a dataclass)."""
    r = S.sched.SearchResult(0, [], [], {"n_configs": 0})
    assert r.status == 0 and r.best_indices == [] and r.pareto_indices == []
    p = S.sched.DPPoint()
    assert p.valid == 0 and len(p.group_of) == 32


def test_split_pick_layout():
    """sched_split_pick: sched_pick + rank + count + 32 split entries."""
    assert C.sizeof(S.sched.SplitPick) == C.sizeof(S.sched.Pick) + 8 + 4 * 32
    r = S.sched.SplitPick()
    assert r.pick.valid == 0 and r.n_clients == 0


def test_split_workspace_and_errors_host():
    """Host-side split setup: count of split vectors (divisor product),
    TOO_LARGE when a split exceeds 32 clients, INVALID for a windowed query."""
    prof = make_profile(3, levels=(50, 100), seed=2)
    q = Query(3, 2, 8, (50, 100), PER_GPU, ((1, 1),))
    sch = S.Scheduler(prof)
    cq = sch.cquery(q)
    n = C.c_size_t()
    ns = C.c_uint32()
    t = np.array([4, 6, 1], np.int32)
    tp = t.ctypes.data_as(C.POINTER(C.c_int32))
    assert S.lib().sched_split_workspace_size(sch._h, C.byref(cq), tp, None, C.byref(n), C.byref(ns)) == 0
    assert ns.value == 3 * 4 * 1 and n.value > 0
    big = np.array([32, 2, 1], np.int32)
    assert S.lib().sched_split_workspace_size(sch._h, C.byref(cq), big.ctypes.data_as(C.POINTER(C.c_int32)),
                                              None, C.byref(n), C.byref(ns)) == S.sched.SCHED_E_TOO_LARGE
    cap = np.array([2, 2, 1], np.int32)
    assert S.lib().sched_split_workspace_size(sch._h, C.byref(cq), big.ctypes.data_as(C.POINTER(C.c_int32)),
                                              cap.ctypes.data_as(C.POINTER(C.c_int32)), C.byref(n),
                                              C.byref(ns)) == 0 and ns.value == 4
    cw = sch.cquery(q.with_range(0, 10))
    assert S.lib().sched_split_workspace_size(sch._h, C.byref(cw), tp, None, C.byref(n),
                                              C.byref(ns)) == S.sched.SCHED_E_INVALID


@pytest.mark.skipif(__import__("torch").cuda.is_available(), reason="checks the no-device path")
def test_no_device_no_fallback():
    """Without a GPU every compute entry point returns SCHED_E_NODEVICE before
    touching the workspace: there is no CPU fallback."""
    prof, q = config("c1")
    sch = S.Scheduler(prof)
    cq = sch.cquery(q)
    fake = C.c_void_p(0x1000)   # never dereferenced
    best = (S.sched.Pick * 4)()
    par = (S.sched.Pick * 16)()
    npar = C.c_uint64()
    rc = S.lib().sched_search(sch._h, C.byref(cq), fake, C.c_size_t(1 << 30), None, best, par,
                              C.c_uint64(16), C.byref(npar), None)
    assert rc == S.sched.SCHED_E_NODEVICE
    dp = (S.sched.DPPoint * 4)()
    fr = (S.sched.DPPoint * 16)()
    rc = S.lib().sched_front_dp(sch._h, C.byref(cq), fake, C.c_size_t(1 << 30), None, dp, fr,
                                C.c_uint64(16), C.byref(npar), None)
    assert rc == S.sched.SCHED_E_NODEVICE
    t = np.array([2, 2, 1, 1], np.int32)
    sb = (S.sched.SplitPick * 4)()
    sp = (S.sched.SplitPick * 16)()
    rc = S.lib().sched_search_splits(sch._h, C.byref(cq), t.ctypes.data_as(C.POINTER(C.c_int32)), None,
                                     fake, C.c_size_t(1 << 30), None, sb, sp, C.c_uint64(16),
                                     C.byref(npar), None)
    assert rc == S.sched.SCHED_E_NODEVICE
    assert S.lib().sched_strerror(S.sched.SCHED_E_NODEVICE)


@pytest.mark.parametrize("scope", [PER_GPU, PER_CLIENT])
def test_rank_rejects_out_of_range_groups_and_levels(scope):
    """sched_rank validates every group id / level digit before using it as
    an index (a group id >= 32 once wrote past a stack buffer)."""
    q = Query(6, 4, 6, (25, 50, 75, 100), scope, ())
    for a, lv in [([0, 40, 0, 1, 1, 2], [0] * 6), ([0, -1, 0, 1, 1, 2], [0] * 6),
                  ([0, 1, 2, 3, 4, 0], [0] * 6),            # group 4 >= G = 4
                  ([0, 0, 1, 1, 2, 2], [0, 0, 1, 1, 4, 4]),   # level digit 4 >= L
                  ([0, 0, 1, 1, 2, 2], [0, 0, 1, 1, -1, -1]),
                  ([0, 127, 0, 0, 0, 0], [0] * 6)]:
        with pytest.raises(S.SchedError) as e:
            S.rank(q, a, lv)
        assert e.value.status == S.sched.SCHED_E_INVALID
    assert S.rank(q, [0, 0, 1, 1, 2, 2], [1, 1, 2, 2, 3, 3] if scope == PER_GPU else [1, 2, 3, 0, 1, 2]) >= 0


def _heuristic_cases():
    rnd = random.Random(2024)
    cases = []
    for k in range(220):
        n = rnd.randint(2, 12)
        g = rnd.randint(1, 8)
        c = rnd.randint(1, n)
        lv = tuple(sorted(rnd.sample((25, 50, 75, 100), rnd.randint(1, 4))))
        scope = rnd.choice((PER_GPU, PER_CLIENT))
        if scope == PER_CLIENT and n > 9:
            scope = PER_GPU
        arch = None
        if k % 5 == 0:   # memory-heavy mixes (WarpX, BerkeleyGW rows) exercise criterion 3
            arch = [rnd.choice((2, 11, 12, 0, 3, 5)) for _ in range(n)]
        cases.append((k, n, g, c, lv, scope, arch))
    return cases


def test_heuristic_equals_oracle_transcription():
    """N2 parity: sched_heuristic returns exactly O6's schedule
    (oracle/heuristic.py, criteria 1-4 of PAPER.md L89-L92, reading R25) --
    group_of, level_of, index and fp64 score, or both report no schedule --
    on 220 seeded queues x both priorities (n = 2..12, G = 1..8, every C,
    level subsets, both scopes, memory-heavy mixes)."""
    from oracle import heuristic as H
    W2 = ((1, 1), (1, 0), (0, 1))
    n_sched = n_none = 0
    for k, n, g, c, lv, scope, arch in _heuristic_cases():
        prof = make_profile(n, levels=(25, 50, 75, 100), seed=900 + k, archetypes=arch)
        q = Query(n, g, c, lv, scope, W2, True)
        sch = S.Scheduler(prof)
        for pr in ("throughput", "energy"):
            w = k % 3
            ref = H.heuristic(prof, q, pr, w=w)
            if ref is None:
                with pytest.raises(S.SchedError) as e:
                    sch.heuristic(q, pr, w)
                assert e.value.status == S.sched.SCHED_E_INFEASIBLE
                n_none += 1
                continue
            a, lvl, idx, pick = sch.heuristic(q, pr, w)
            assert (a, lvl, idx) == (ref["rgs"], ref["level_of"], ref["index"]), (k, pr)
            assert bool(pick.valid) == ref["feasible"]
            if ref["feasible"]:
                assert (pick.makespan_s, pick.energy_j, pick.score64) == (ref["T"], ref["E"], ref["score64"])
            n_sched += 1
        sch.close()
    assert n_sched >= 250 and n_none >= 5


@pytest.mark.parametrize("name", list(CONFIGS))
def test_heuristic_equals_oracle_transcription_configs(name):
    from oracle import heuristic as H
    prof, q = config(name)
    sch = S.Scheduler(prof)
    for pr in ("throughput", "energy"):
        for w in range(len(q.weights)):
            ref = H.heuristic(prof, q, pr, w=w)
            if ref is None:
                with pytest.raises(S.SchedError):
                    sch.heuristic(q, pr, w)
                continue
            a, lvl, idx, pick = sch.heuristic(q, pr, w)
            assert (a, lvl, idx) == (ref["rgs"], ref["level_of"], ref["index"])
            assert bool(pick.valid) == ref["feasible"]
            if ref["feasible"]:
                assert pick.score64 == ref["score64"]
