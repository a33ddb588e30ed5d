"""CPU oracle for the exhaustive co-scheduling configuration search.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` legs may import this package.  It shares no
code with the CUDA path (paper_conf_sc_weaverkmeh0m24_b200/) and neither
imports the other; both consume the seeded inputs of synth/.

  counts.py  closed-form |Omega| (Stirling / Bell / EGF)        [pinned]
  brute.py   O2: all G^N labelings -> canonical RGS, sort order,  [pinned]
             pure-Python fp64 score (N <= 6)
  enum.c     O1: recursive fp64 enumerator, index windows        [pinned]
             (ctypes wrapper below; parallel windows + merge)
  dpcert.c   O3/O4: exact subset-DP certificate of optimal values
  split.py   O5: scheduling-configuration (task split) search over the
             split vectors of the queue (R29)

Every function above is pinned by tests that do not re-type it (closed forms,
brute force, hand-derived configurations, the paper's Table II/III numbers).
Parity unpinned: whether the model's predicted X, Y agree with the paper's
MEASURED Figs 2-5 -- the paper prints neither a prediction model nor numbers
for those figures.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from concurrent.futures import ProcessPoolExecutor

import numpy as np

from . import counts  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "enum.c")
_SRCS = [_SRC, os.path.join(_HERE, "dpcert.c")]
_lib = None

ORACLE_CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-msse2",
                 "-mfpmath=sse", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or any(os.path.getmtime(_SO) < os.path.getmtime(x) for x in _SRCS):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *ORACLE_CFLAGS, "-o", tmp, *_SRCS])
        os.replace(tmp, _SO)
    return _SO


class _Profile(C.Structure):
    _fields_ = [("n", C.c_int), ("lp", C.c_int), ("level_pct", C.POINTER(C.c_int)),
                ("t", C.POINTER(C.c_float)), ("p", C.POINTER(C.c_float)),
                ("u", C.POINTER(C.c_float)), ("bw", C.POINTER(C.c_float)),
                ("mem", C.POINTER(C.c_int)), ("d", C.POINTER(C.c_float)),
                ("mem_cap", C.c_int), ("ps", C.c_float)]


class _Query(C.Structure):
    _fields_ = [("n", C.c_int), ("g", C.c_int), ("c", C.c_int), ("L", C.c_int),
                ("lev", C.POINTER(C.c_int)), ("scope", C.c_int), ("nw", C.c_int),
                ("wa", C.POINTER(C.c_int)), ("wb", C.POINTER(C.c_int)),
                ("lo", C.c_uint64), ("hi", C.c_uint64), ("want_pareto", C.c_int),
                ("model", C.c_uint), ("power_cap", C.c_float),
                ("tseq_base", C.c_double), ("eseq_base", C.c_double)]


class _Best(C.Structure):
    _fields_ = [("idx", C.c_uint64), ("f", C.c_double), ("t", C.c_double),
                ("e", C.c_double), ("found", C.c_int)]


class _Point(C.Structure):
    _fields_ = [("idx", C.c_uint64), ("t", C.c_double), ("e", C.c_double)]


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _lib.oracle_search.restype = C.c_int
        _lib.oracle_config.restype = C.c_int
        _lib.oracle_score_config.restype = C.c_int
        _lib.oracle_objective.restype = C.c_double
        _lib.oracle_objective.argtypes = [C.c_double] * 4 + [C.c_int] * 2
    return _lib


def _ptr(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


class _Pack:
    """Keeps numpy buffers alive while the C structs point at them."""

    def __init__(self, prof, q):
        self.keep = []

        def arr(x, dt):
            a = np.ascontiguousarray(x, dtype=dt)
            self.keep.append(a)
            return a
        lp = prof.n_levels
        self.P = _Profile(prof.n_workflows, lp, _ptr(arr(prof.level_pct, np.int32), C.c_int),
                          _ptr(arr(prof.solo_time_s, np.float32), C.c_float),
                          _ptr(arr(prof.solo_power_w, np.float32), C.c_float),
                          _ptr(arr(prof.sm_util, np.float32), C.c_float),
                          _ptr(arr(prof.bw_util, np.float32), C.c_float),
                          _ptr(arr(prof.max_mem_mib, np.int32), C.c_int),
                          _ptr(arr(prof.corun_slowdown, np.float32), C.c_float),
                          int(prof.mem_capacity_mib), float(prof.static_power_w))
        pct = [int(x) for x in prof.level_pct]
        self.lev_idx = [pct.index(int(v)) for v in q.levels]
        self.l100 = pct.index(100)
        lev = arr(self.lev_idx, np.int32)
        wa = arr([w[0] for w in q.weights] or [0], np.int32)
        wb = arr([w[1] for w in q.weights] or [0], np.int32)
        hi = q.index_hi if q.index_hi is not None else count(q)
        self.Q = _Query(q.n, q.g, min(q.c, q.n), len(q.levels), _ptr(lev, C.c_int),
                        q.scope, len(q.weights), _ptr(wa, C.c_int), _ptr(wb, C.c_int),
                        int(q.index_lo), int(hi), int(bool(q.want_pareto)),
                        int(getattr(q, "model", 0)), float(getattr(q, "power_cap", 0.0)),
                        float(getattr(q, "tseq_base", 0.0)), float(getattr(q, "eseq_base", 0.0)))


def count(q) -> int:
    """|Omega| via the oracle's memoised recursion (u128)."""
    lo = C.c_uint64()
    hi = C.c_uint64()
    lev = np.zeros(max(1, len(q.levels)), np.int32)
    w = np.zeros(1, np.int32)
    Q = _Query(q.n, q.g, min(q.c, q.n), len(q.levels), _ptr(lev, C.c_int), q.scope, 0,
               _ptr(w, C.c_int), _ptr(w, C.c_int), 0, 0, 0)
    lib().oracle_count(C.byref(Q), C.byref(lo), C.byref(hi))
    return (hi.value << 64) | lo.value


def constants(prof, q):
    pk = _Pack(prof, q)
    ts = C.c_double()
    es = C.c_double()
    lib().oracle_constants(C.byref(pk.P), C.byref(pk.Q), pk.l100, C.byref(ts), C.byref(es))
    return ts.value, es.value


def search(prof, q, pareto_cap: int = 1 << 16) -> dict:
    """Exhaustive fp64 search of the window [q.index_lo, q.index_hi)."""
    pk = _Pack(prof, q)
    nw = len(q.weights)
    best = (_Best * max(1, nw))()
    par = (_Point * pareto_cap)()
    npar = C.c_int()
    ncfg = C.c_uint64()
    nfeas = C.c_uint64()
    rc = lib().oracle_search(C.byref(pk.P), C.byref(pk.Q), pk.l100, best, par, pareto_cap,
                             C.byref(npar), C.byref(ncfg), C.byref(nfeas))
    if rc != 0:
        raise RuntimeError("oracle Pareto capacity overflow")
    out_best = [(best[w].idx, best[w].f, best[w].t, best[w].e) if best[w].found else None
                for w in range(nw)]
    pts = sorted([(par[i].idx, par[i].t, par[i].e) for i in range(npar.value)],
                 key=lambda x: (x[1], x[2], x[0]))
    ts, es = constants(prof, q)
    return dict(best=out_best, pareto=pts if q.want_pareto else [],
                nconfigs=ncfg.value, nfeasible=nfeas.value, tseq=ts, eseq=es)


def merge(parts, want_pareto=True) -> dict:
    """Merge window results: best = max F, ties lowest index; Pareto = exact filter."""
    nw = len(parts[0]["best"])
    best = []
    for w in range(nw):
        b = None
        for p in parts:
            x = p["best"][w]
            if x is None:
                continue
            if b is None or x[1] > b[1] or (x[1] == b[1] and x[0] < b[0]):
                b = x
        best.append(b)
    pts = []
    if want_pareto:
        allp = sorted([x for p in parts for x in p["pareto"]], key=lambda x: (x[1], x[2], x[0]))
        bestE = None
        for x in allp:                # T ascending, then E ascending, then idx
            if bestE is None or x[2] < bestE:
                pts.append(x)
                bestE = x[2]
    return dict(best=best, pareto=pts, nconfigs=sum(p["nconfigs"] for p in parts),
                nfeasible=sum(p["nfeasible"] for p in parts),
                tseq=parts[0]["tseq"], eseq=parts[0]["eseq"])


def _search_star(args):
    return search(*args)


def search_parallel(prof, q, procs: int | None = None, windows: int | None = None,
                    pareto_cap: int = 1 << 16) -> dict:
    """Process pool over disjoint index windows, merged with `merge`."""
    hi = q.index_hi if q.index_hi is not None else count(q)
    lo = q.index_lo
    procs = procs or os.cpu_count() or 1
    windows = windows or procs * 4
    step = max(1, -(-(hi - lo) // windows))
    qs = [q.with_range(a, min(hi, a + step)) for a in range(lo, hi, step)]
    if procs == 1 or len(qs) == 1:
        parts = [search(prof, x, pareto_cap) for x in qs]
    else:
        with ProcessPoolExecutor(procs) as ex:
            parts = list(ex.map(_search_star, [(prof, x, pareto_cap) for x in qs]))
    return merge(parts, q.want_pareto)


def score_window(prof, q):
    """fp64 canonical (T, E) of every configuration of [q.index_lo,
    q.index_hi) in index order (NaN where infeasible): two numpy arrays."""
    pk = _Pack(prof, q)
    n = int(pk.Q.hi - pk.Q.lo)
    T = np.empty(n, np.float64)
    E = np.empty(n, np.float64)
    f = lib().oracle_score_window
    f.restype = C.c_uint64
    got = f(C.byref(pk.P), C.byref(pk.Q), _ptr(T, C.c_double), _ptr(E, C.c_double))
    assert got == n
    return T, E


def config(q, idx: int):
    """Index -> (RGS a[n], level digits) by the oracle's own enumeration."""
    a = (C.c_int * 64)()
    lv = (C.c_int * 64)()
    lev = np.zeros(max(1, len(q.levels)), np.int32)
    w = np.zeros(1, np.int32)
    Q = _Query(q.n, q.g, min(q.c, q.n), len(q.levels), _ptr(lev, C.c_int), q.scope, 0,
               _ptr(w, C.c_int), _ptr(w, C.c_int), 0, 0, 0)
    k = lib().oracle_config(C.byref(Q), C.c_uint64(idx), a, lv)
    if k < 0:
        raise IndexError(idx)
    nd = q.n if q.scope == 0 else k
    return [a[i] for i in range(q.n)], [lv[j] for j in range(nd)]


def score(prof, q, rgs, digits):
    """(feasible, T, E) of one configuration, fp64 canonical order."""
    pk = _Pack(prof, q)
    k = max(rgs) + 1
    pl = [pk.lev_idx[digits[i] if q.scope == 0 else digits[rgs[i]]] for i in range(q.n)]
    a = (C.c_int * 64)(*rgs)
    plc = (C.c_int * 64)(*pl)
    T = C.c_double()
    E = C.c_double()
    ok = lib().oracle_score_config(C.byref(pk.P), C.byref(pk.Q), q.n, a, k, plc, C.byref(T), C.byref(E))
    return bool(ok), T.value, E.value


def objective(tseq, eseq, T, E, a, b) -> float:
    return lib().oracle_objective(tseq, eseq, T, E, a, b)


def _client_fronts(args):
    """Phase 1 of O4 for groups B in [b_lo, b_hi): (off[b_hi - b_lo + 1], t, e)."""
    prof, q, b_lo, b_hi = args[:4]
    batched = args[4] if len(args) > 4 else 1
    pk = _Pack(prof, q)
    lev = (C.c_int * len(pk.lev_idx))(*pk.lev_idx)
    f = lib().oracle_client_fronts
    f.restype = C.c_longlong
    off = np.zeros(b_hi - b_lo + 1, np.int64)
    cap = 1 << 16
    while True:
        t = np.zeros(cap, np.float64)
        e = np.zeros(cap, np.float64)
        n = f(C.byref(pk.P), q.n, min(q.c, q.n), len(q.levels), lev, C.c_uint(b_lo), C.c_uint(b_hi),
              _ptr(t, C.c_double), _ptr(e, C.c_double), _ptr(off, C.c_longlong), C.c_longlong(cap),
              int(batched))
        if n >= 0:
            return off, t[:n].copy(), e[:n].copy()
        cap *= 4


def _client_tasks(n, c, L, parts):
    """Split [1, 2^n) into ~parts ranges of similar cost (L^|B| |B|^2 per group)."""
    cost = [0.0] * (1 << n)
    for B in range(1, 1 << n):
        s = bin(B).count("1")
        cost[B] = float(L) ** s * (s * s + 4) if s <= c else 0.0
    tot = sum(cost)
    out, lo, acc = [], 0, 0.0
    for B in range(1 << n):
        acc += cost[B]
        if acc >= tot / parts or B == (1 << n) - 1:
            out.append((lo, B + 1))
            lo, acc = B + 1, 0.0
    return out


def client_fronts_parallel(prof, q, procs: int, parts: int | None = None):
    """Phase 1 of O4 over a process pool; returns (off[2^n + 1], t, e)."""
    tasks = _client_tasks(q.n, min(q.c, q.n), len(q.levels), parts or procs * 16)
    # largest tasks first so the pool's tail is short
    order = sorted(range(len(tasks)), key=lambda i: tasks[i][0] - tasks[i][1])
    res = [None] * len(tasks)
    with ProcessPoolExecutor(procs) as ex:
        futs = {i: ex.submit(_client_fronts, (prof, q, *tasks[i])) for i in order}
        for i in order:
            res[i] = futs[i].result()
    offs, ts, es, base = [], [], [], 0
    for off, t, e in res:
        offs.append(off[:-1] + base)
        ts.append(t)
        es.append(e)
        base += t.size
    off = np.concatenate(offs + [np.array([base], np.int64)])
    return off, np.concatenate(ts), np.concatenate(es)


def dp_certificate(prof, q, cap: int = 1 << 20, procs: int = 1):
    """O3 (PER_GPU) / O4 (PER_CLIENT) in dpcert.c: exact Pareto-front values
    [(T, E)] (T ascending) of the whole space and the exact optimum F per
    weight (max over the front, canonical fp64).  Values only, no indices.
    procs > 1 (PER_CLIENT): O4's per-group fronts in a process pool over
    disjoint group ranges, then the same DP (oracle_client_dp)."""
    assert getattr(q, "model", 0) == 0, "certificate covers the canonical model"
    pk = _Pack(prof, q)
    ot = (C.c_double * cap)()
    oe = (C.c_double * cap)()
    lev = (C.c_int * len(pk.lev_idx))(*pk.lev_idx)
    if q.scope == 0 and procs > 1:
        off, t, e = client_fronts_parallel(prof, q, procs)
        nf = lib().oracle_client_dp(q.n, q.g, _ptr(t, C.c_double), _ptr(e, C.c_double),
                                    _ptr(off, C.c_longlong), ot, oe, cap)
    else:
        fn = lib().oracle_dpcert if q.scope == 1 else lib().oracle_dpcert_client   # O3 / O4
        nf = fn(C.byref(pk.P), q.n, q.g, min(q.c, q.n), len(q.levels), lev, ot, oe, cap)
    if nf < 0:
        raise RuntimeError("certificate capacity / size")
    front = [(ot[i], oe[i]) for i in range(nf)]
    ts, es = constants(prof, q)
    best = [max(objective(ts, es, T, E, a, b) for T, E in front) if front else None for a, b in q.weights]
    return dict(front=front, best=best, tseq=ts, eseq=es)
