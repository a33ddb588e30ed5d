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
