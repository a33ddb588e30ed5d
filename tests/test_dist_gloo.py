"""N>1 path on CPU: world-size-2 gloo process group.

Each rank's shard (chunks c with c % R == rank) is scored by the
oracle (there is no GPU here), converted to picks, exchanged with the
product's all_gather + sched_merge (dist.exchange), and the merged result
must equal the oracle's unsharded answer exactly on every rank.
"""
import os
import socket

import pytest
import torch.multiprocessing as mp

import oracle
from synth import Query, make_profile, PER_GPU, PER_CLIENT


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _to_picks(best, pareto, tseq, eseq):
    from paper_conf_sc_weaverkmeh0m24_b200.sched import Pick
    bl = []
    for b in best:
        p = Pick()
        if b is not None:
            p.valid = 1
            p.index, p.score64, p.makespan_s, p.energy_j = b
            p.x64, p.y64 = tseq / b[2], eseq / b[3]
        bl.append(p)
    pl = []
    for idx, T, E in pareto:
        p = Pick()
        p.valid = 1
        p.index, p.makespan_s, p.energy_j = idx, T, E
        pl.append(p)
    return bl, pl


def _worker(rank, world, port, case, out):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_weaverkmeh0m24_b200 import dist as D
    n, g, c, levels, scope, weights, cl = case
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=21)
    q = Query(n, g, c, levels, scope, weights, True)
    tot = oracle.count(q)
    parts = []
    ch = 0
    while (ch << cl) < tot:
        if ch % world == rank:
            parts.append(oracle.search(prof, q.with_range(ch << cl, min(tot, (ch + 1) << cl))))
        ch += 1
    m = oracle.merge(parts) if parts else None
    ts, es = oracle.constants(prof, q)
    best, par = _to_picks(m["best"] if m else [None] * len(weights), m["pareto"] if m else [], ts, es)
    mb, mpar, nbytes = D.exchange(best, par, len(weights))
    out[rank] = ([(b.index, b.score64) if b.valid else None for b in mb],
                 [(p.index, p.makespan_s, p.energy_j) for p in mpar], nbytes)
    dist.destroy_process_group()


@pytest.mark.parametrize("case", [
    (7, 3, 4, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1), (1, 0)), 12),
    (6, 3, 6, (50, 100), PER_CLIENT, ((0, 1), (1, 2)), 12),
])
def test_gloo_world2_exchange_merge(case):
    world = 2
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(world, port, case, out), nprocs=world, join=True)
    n, g, c, levels, scope, weights, _ = case
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=21)
    q = Query(n, g, c, levels, scope, weights, True)
    ref = oracle.search(prof, q)
    exp_best = [(b[0], b[1]) if b else None for b in ref["best"]]
    for r in range(world):
        best, par, nbytes = out[r]
        assert best == exp_best
        assert par == ref["pareto"]
        assert nbytes > 0


class _OracleShardSched:
    """Stands in for Scheduler on CPU: search(q, shard=(r, R), chunk_log2)
    scores the shard's chunks with the oracle (drop > 0: the shard's first
    chunk loses its last `drop` indices -- fault injection)."""

    def __init__(self, prof, drop=0):
        self.prof, self.drop = prof, drop

    def search(self, q, shard=(0, 1), chunk_log2=24, **kw):
        from paper_conf_sc_weaverkmeh0m24_b200.sched import SearchResult
        r, R = shard
        tot = oracle.count(q)
        parts, ch, first = [], 0, True
        while (ch << chunk_log2) < tot:
            if ch % R == r:
                hi = min(tot, (ch + 1) << chunk_log2)
                if first and self.drop:
                    hi -= self.drop
                first = False
                parts.append(oracle.search(self.prof, q.with_range(ch << chunk_log2, hi)))
            ch += 1
        m = oracle.merge(parts) if parts else None
        ts, es = oracle.constants(self.prof, q)
        best, par = _to_picks(m["best"] if m else [None] * len(q.weights), m["pareto"] if m else [], ts, es)
        return SearchResult(0, best, par, {"n_configs": m["nconfigs"] if m else 0})


def _sharded_worker(rank, world, port, drop, slices, out):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sc_weaverkmeh0m24_b200 import dist as D
    prof = make_profile(7, levels=(25, 50, 75, 100), seed=22)
    q = Query(7, 3, 4, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1)), True)
    try:
        best, par, res, n_all = D.sharded_search(_OracleShardSched(prof, drop if rank == 1 else 0), q,
                                                 chunk_log2=6, slices=slices, total=oracle.count(q))
        out[rank] = ("ok", [(b.index, b.score64) for b in best],
                     [(p.index, p.makespan_s, p.energy_j) for p in par], n_all)
    except D.CoverageError as e:
        out[rank] = ("coverage", str(e))
    dist.destroy_process_group()


@pytest.mark.parametrize("drop", [0, 3])
def test_gloo_world2_sharded_search_coverage(drop):
    """dist.sharded_search at world 2: exchange + merge equal the unsharded
    oracle and the all-reduced scored count equals |Omega|; a rank that
    silently loses 3 indices raises CoverageError on every rank."""
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_sharded_worker, args=(2, _free_port(), drop, (0, 1), out), nprocs=2, join=True)
    prof = make_profile(7, levels=(25, 50, 75, 100), seed=22)
    q = Query(7, 3, 4, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1)), True)
    ref = oracle.search(prof, q)
    for r in range(2):
        if drop:
            assert out[r][0] == "coverage"
        else:
            st, best, par, n_all = out[r]
            assert best == [(b[0], b[1]) for b in ref["best"]] and par == ref["pareto"]
            assert n_all == ref["nconfigs"] == oracle.count(q)


def test_slice_index_count_matches_enumeration():
    from paper_conf_sc_weaverkmeh0m24_b200.dist import slice_index_count
    for lo, hi, cl, R in [(0, 1000, 4, 3), (17, 999, 3, 5), (5, 6, 2, 2), (0, 0, 4, 2), (100, 613, 5, 64)]:
        for r in range(R):
            assert slice_index_count(lo, hi, cl, r, R) == sum(1 for i in range(lo, hi) if (i >> cl) % R == r)
