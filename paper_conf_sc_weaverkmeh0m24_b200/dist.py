"""Multi-GPU layer: one process per GPU, index space split
by chunks (chunk c -> rank c mod R, inside sched_search), per-rank results
exchanged with two all_gathers over the process group (NCCL over NVLink on
the box; gloo in the CPU tests) and merged exactly by sched_merge on every
rank.  The merged result is independent of the rank count.
"""
from __future__ import annotations

import ctypes as C

import numpy as np
import torch
import torch.distributed as dist

from .sched import Pick, merge

PICK_BYTES = C.sizeof(Pick)


def picks_to_array(picks) -> np.ndarray:
    buf = (Pick * max(1, len(picks)))(*picks)
    return np.frombuffer(bytes(buf), dtype=np.uint8)[: PICK_BYTES * len(picks)].copy()


def array_to_picks(a: np.ndarray):
    n = a.size // PICK_BYTES
    if n == 0:
        return []
    buf = (Pick * n).from_buffer_copy(a[: n * PICK_BYTES].tobytes())
    return [buf[i] for i in range(n)]


def exchange(best, pareto, n_weights, group=None, device=None, pareto_cap=1 << 16):
    """All-gather every rank's (best[W], pareto) records and merge them exactly.

    Two collectives: (1) per-rank Pareto counts; (2) fixed-size records
    [W best | max-count Pareto, zero-padded].  Returns (best, pareto, bytes).
    """
    world = dist.get_world_size(group)
    dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                             if dist.get_backend(group) == "nccl" else torch.device("cpu"))
    cnt = torch.tensor([len(pareto)], dtype=torch.int64, device=dev)
    cnts = torch.empty(world, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(cnts, cnt, group=group)
    counts = [int(x) for x in cnts.cpu()]
    mx = max(counts)
    rec = np.zeros(PICK_BYTES * (n_weights + mx), dtype=np.uint8)
    b = picks_to_array(best)
    rec[: b.size] = b
    p = picks_to_array(pareto)
    rec[PICK_BYTES * n_weights: PICK_BYTES * n_weights + p.size] = p
    mine = torch.from_numpy(rec).to(dev)
    allr = torch.empty(world * rec.size, dtype=torch.uint8, device=dev)
    dist.all_gather_into_tensor(allr, mine, group=group)
    host = allr.cpu().numpy().reshape(world, rec.size)
    rank_best, rank_par = [], []
    for r in range(world):
        rank_best.append(array_to_picks(host[r, : PICK_BYTES * n_weights]))
        rank_par.append(array_to_picks(host[r, PICK_BYTES * n_weights: PICK_BYTES * (n_weights + counts[r])]))
    mb, mp = merge(rank_best, rank_par, n_weights, pareto_cap)
    return mb, mp, int(allr.numel() + cnts.numel() * 8)


class CoverageError(RuntimeError):
    pass


def slice_index_count(lo: int, hi: int, chunk_log2: int, r: int, R: int) -> int:
    """Number of indices i in [lo, hi) whose chunk (i >> chunk_log2) is
    congruent to r mod R: the share of shard (r, R)."""
    def upto(x):
        c = x >> chunk_log2
        full, m = divmod(c, R)
        n = full << chunk_log2
        if m > r:
            n += 1 << chunk_log2
        elif m == r:
            n += x & ((1 << chunk_log2) - 1)
        return n
    return upto(hi) - upto(lo)


def check_coverage(n_scored: int, lo: int, hi: int, chunk_log2: int, s_idx: int, s_cnt: int,
                   world: int) -> int:
    """Sum over ranks of the scored configurations must equal the index count
    of the searched slice (coverage = |range|); raises otherwise.
    Rank r of `world` searches shard (s_idx * world + r, s_cnt * world)."""
    expect = sum(slice_index_count(lo, hi, chunk_log2, s_idx * world + r, s_cnt * world) for r in range(world))
    if n_scored != expect:
        raise CoverageError(f"ranks scored {n_scored} configurations, slice ({s_idx}/{s_cnt}) of "
                            f"[{lo}, {hi}) over {world} ranks has {expect}")
    return expect


def allreduce_sum(x: int, group=None, device=None) -> int:
    dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                             if dist.get_backend(group) == "nccl" else torch.device("cpu"))
    t = torch.tensor([int(x)], dtype=torch.int64, device=dev)
    dist.all_reduce(t, group=group)
    return int(t.item())


def sharded_search(sched, q, group=None, chunk_log2=24, slices=(0, 1), total=None, **kw):
    """This rank's share of q (optionally one of `slices[1]` cyclic slices of
    the chunk sequence), then exchange + exact merge.  The configurations
    scored by all ranks are summed (all_reduce) and checked against the
    slice's index count (CoverageError on a mismatch: a lost or truncated
    shard never yields an 'optimum').  total: |Omega| (default: count(q)).
    Returns (best, pareto, local SearchResult, n_configs summed over ranks)."""
    from .sched import count
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    s_idx, s_cnt = slices
    res = sched.search(q, shard=(s_idx * world + rank, s_cnt * world), chunk_log2=chunk_log2, **kw)
    best, pareto, _ = exchange(res.best, res.pareto, len(q.weights), group=group)
    n_all = allreduce_sum(res.stats["n_configs"], group=group)
    tot = count(q) if total is None else total
    hi = tot if q.index_hi is None else min(int(q.index_hi), tot)
    check_coverage(n_all, int(q.index_lo), hi, chunk_log2, s_idx, s_cnt, world)
    return best, pareto, res, n_all
