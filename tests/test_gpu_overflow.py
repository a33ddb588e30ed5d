"""Candidate-buffer overflow and the re-run passes:
a search whose candidate buffer overflows stops the pass early and re-runs
it (pass 2 re-bucketed to the overflowing pass's candidate span with a fresh
staircase; pass 3 reseeded).  Forced here with small `candidate_cap`s: the
result must equal the oracle on oracle-sized windows, and, on seeded
bench-size slices (>= 2^32 configurations), the default-capacity search."""
import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, Query
from test_gpu_parity import check

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name,scope,lo", [
    ("c4", None, 123_456_789_012),          # tile kernel
    ("c3", 0, 9_876_543_210),               # literal per-client c3: k_ctile2
    ("c5", None, 301_234_567_891),          # suffix kernel
])
@pytest.mark.parametrize("cap", [64, 512])
def test_small_candidate_buffer_windows(name, scope, lo, cap):
    """SCHED_E_CAPACITY is a legitimate outcome only when the default search
    itself emits more candidates than the small buffer holds; any other
    outcome must be the oracle's answer bitwise."""
    prof, q = config(name)
    if scope is not None:
        q = Query(q.n, q.g, q.c, q.levels, scope, q.weights, q.want_pareto)
    qw = q.with_range(lo, lo + 3_000_000)
    sch = S.Scheduler(prof)
    res = sch.search(qw, candidate_cap=cap, allow_capacity=True)
    if res.status == S.sched.SCHED_E_CAPACITY:
        assert sch.search(qw).stats["n_candidates"] > cap
        return
    check(res, oracle.search(prof, qw), qw)


@pytest.mark.parametrize("name,scope,cap", [("c4", None, 1 << 14), ("c3", 0, 1 << 15), ("c5", None, 1 << 12)])
def test_small_candidate_buffer_seeded_slices(name, scope, cap):
    """Seeded searches (a 1/64 chunk slice: >= 2^32 configurations) with a
    candidate buffer small enough to overflow: the same best picks and Pareto
    set as the default-capacity search of the same slice."""
    prof, q = config(name)
    if scope is not None:
        q = Query(q.n, q.g, q.c, q.levels, scope, q.weights, q.want_pareto)
    sch = S.Scheduler(prof)
    kw = {"shard": (5, 64), "chunk_log2": 24} if name != "c5" else {}
    ref = sch.search(q, **kw)
    res = sch.search(q, candidate_cap=cap, allow_capacity=True, **kw)
    assert res.stats["n_configs"] == ref.stats["n_configs"]
    if res.status == S.sched.SCHED_E_CAPACITY:  # every re-run overflowed too: reported, never a wrong answer
        assert ref.stats["n_candidates"] > cap
        return
    assert [(b.index, b.score64) for b in res.best] == [(b.index, b.score64) for b in ref.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in res.pareto] == \
        [(p.index, p.makespan_s, p.energy_j) for p in ref.pareto]
