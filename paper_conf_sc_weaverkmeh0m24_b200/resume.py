"""Checkpoint / resume and coverage for long exhaustive searches (SURVEY 5
"failure detection", "checkpoint / resume"; the c4 search is 43 s on one
B200, a per-client space far longer).

The search is restartable by index range (include/sched.h index_lo/hi), and
its partial results are tiny (W best picks + a Pareto list), so a search is
cut into contiguous index windows, each searched by `sched_search` and its
result appended as one JSON line to a checkpoint file (floats as hex:
bit-exact).  A restart skips the windows already recorded for the same
profile and query (SHA-256 fingerprint); the final result is the exact
`sched_merge` of all windows, equal to a one-shot search.  Coverage is
checked before merging: the recorded windows must tile [0, |Omega|) exactly
and their configuration counts must sum to |Omega|; a lost or truncated
window raises CoverageError instead of returning a partial optimum.
"""
from __future__ import annotations

import dataclasses
import hashlib
import json
import os
import warnings

import numpy as np

from .sched import Pick, count, merge


class CoverageError(RuntimeError):
    pass


_PICK_F = [f for f, _ in Pick._fields_]


def pick_to_json(p: Pick) -> dict:
    return {f: (float(getattr(p, f)).hex() if isinstance(getattr(p, f), float) else int(getattr(p, f)))
            for f in _PICK_F}


def pick_from_json(d: dict) -> Pick:
    p = Pick()
    for f in _PICK_F:
        v = d[f]
        setattr(p, f, float.fromhex(v) if isinstance(v, str) else v)
    return p


def fingerprint(profile, q) -> str:
    """SHA-256 over the profile tables and the query fields that define the
    space and the objectives (not the index window)."""
    h = hashlib.sha256()
    for name in ("level_pct", "solo_time_s", "solo_power_w", "sm_util", "bw_util", "max_mem_mib",
                 "corun_slowdown"):
        a = np.ascontiguousarray(getattr(profile, name))
        h.update(name.encode())
        h.update(str(a.dtype).encode())
        h.update(a.tobytes())
    h.update(repr((int(profile.mem_capacity_mib), float(profile.static_power_w))).encode())
    qd = dataclasses.asdict(dataclasses.replace(q, index_lo=0, index_hi=None))
    h.update(json.dumps(qd, sort_keys=True, default=str).encode())
    return h.hexdigest()


def windows_of(total: int, n_windows: int, align: int = 1 << 24):
    """[lo, hi) windows tiling [0, total), boundaries on multiples of `align`
    (the chunk size) where the space allows."""
    n_windows = max(1, n_windows)
    step = -(-total // n_windows)
    step = max(align, -(-step // align) * align)
    return [(lo, min(lo + step, total)) for lo in range(0, total, step)] or [(0, 0)]


def load(path: str, fp: str) -> dict:
    """{(lo, hi): record} of the checkpoint's records for this fingerprint
    (records of other searches and a torn last line are ignored)."""
    done = {}
    if not os.path.exists(path):
        return done
    with open(path) as f:
        for line in f:
            try:
                r = json.loads(line)
            except json.JSONDecodeError:
                continue
            if r.get("fp") == fp:
                done[(r["lo"], r["hi"])] = r
    return done


def check_coverage(records, total: int) -> None:
    spans = sorted((r["lo"], r["hi"]) for r in records)
    pos = 0
    for lo, hi in spans:
        if lo != pos:
            raise CoverageError(f"index range [{pos}, {lo}) not covered")
        pos = hi
    if pos != total:
        raise CoverageError(f"index range [{pos}, {total}) not covered")
    n = sum(int(r["n_configs"]) for r in records)
    if n != total:
        raise CoverageError(f"windows scored {n} configurations, the space has {total}")


def search_resumable(sched, profile, q, path: str, n_windows: int = 64, max_windows: int | None = None,
                     search_fn=None, pareto_cap: int = 1 << 16, align: int = 1 << 24):
    """Exhaustive search of the whole space of `q`, checkpointed per window.

    sched: a Scheduler for `profile`.  search_fn(qw) -> SearchResult-like
    (best, pareto, stats["n_configs"]); default sched.search.  align: window
    boundaries on multiples of this (default the 2^24 chunk).  max_windows:
    stop after searching that many NEW windows (simulates an interrupted
    run); returns None then.  Otherwise returns (best[W], pareto, stats)
    with stats = {"n_configs", "n_feasible", "windows", "resumed"}.
    """
    fp = fingerprint(profile, q)
    total = count(q)
    done = load(path, fp)
    search = search_fn if search_fn is not None else (lambda qw: sched.search(qw, pareto_cap=pareto_cap))
    new = 0
    wins = windows_of(total, n_windows, align)
    # only records of the current window split count as resumed; records of
    # another split (n_windows / align changed) are ignored, not merged
    resumed = sum(1 for w in wins if w in done)
    stale = len(done) - resumed
    if stale:
        warnings.warn(f"{path}: {stale} checkpoint record(s) of another window split "
                      f"(n_windows={n_windows}, align={align} now) are ignored", RuntimeWarning)
    for lo, hi in wins:
        if (lo, hi) in done:
            continue
        if max_windows is not None and new >= max_windows:
            return None
        res = search(q.with_range(lo, hi))
        rec = {"fp": fp, "lo": lo, "hi": hi, "n_windows": n_windows, "align": align,
               "n_configs": int(res.stats["n_configs"]),
               "n_feasible": int(res.stats["n_feasible"]),
               "best": [pick_to_json(b) for b in res.best],
               "pareto": [pick_to_json(p) for p in res.pareto]}
        with open(path, "a") as f:
            f.write(json.dumps(rec) + "\n")
            f.flush()
            os.fsync(f.fileno())
        done[(lo, hi)] = rec
        new += 1
    recs = [done[w] for w in wins]   # records of another window split are not mixed in
    check_coverage(recs, total)
    nw = len(q.weights)
    rank_best = [[pick_from_json(b) for b in r["best"]] if r["best"] else [Pick() for _ in range(nw)]
                 for r in recs]
    rank_par = [[pick_from_json(p) for p in r["pareto"]] for r in recs]
    best, par = merge(rank_best, rank_par, nw, pareto_cap)
    return best, par, {"n_configs": sum(r["n_configs"] for r in recs),
                       "n_feasible": sum(r["n_feasible"] for r in recs),
                       "windows": len(recs), "resumed": resumed, "stale": stale}
