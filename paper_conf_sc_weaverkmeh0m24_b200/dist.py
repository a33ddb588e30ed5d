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


def sharded_search(sched, q, group=None, chunk_log2=24, slices=(0, 1), **kw):
    """This rank's share of q (optionally one of `slices[1]` cyclic slices of
    the chunk sequence), then exchange + exact merge.  Returns
    (best, pareto, local SearchResult, n_configs summed over ranks)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    s_idx, s_cnt = slices
    res = sched.search(q, shard=(s_idx * world + rank, s_cnt * world), chunk_log2=chunk_log2, **kw)
    best, pareto, _ = exchange(res.best, res.pareto, len(q.weights), group=group)
    return best, pareto, res
