"""Thin Python binding of include/sched.h (argument marshalling only).

Every step of the search runs in libsched.so's CUDA kernels; PyTorch is
used only for the caller-owned device workspace and the CUDA stream.
There is no CPU fallback: a missing libsched.so or a missing GPU raises.
"""
from __future__ import annotations

import ctypes as C
import dataclasses
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("SCHED_SO_PATH") or os.path.join(_HERE, "libsched.so")  # override: A/B measurements

SCHED_OK = 0
SCHED_E_INVALID = -1
SCHED_E_TOO_LARGE = -2
SCHED_E_CUDA = -3
SCHED_E_CAPACITY = -4
SCHED_E_INFEASIBLE = -5
SCHED_E_WORKSPACE = -6
SCHED_E_NODEVICE = -7
PER_CLIENT = 0
PER_GPU = 1
SCHED_MODEL_COUNT_IDLE = 1        # scoring-model variants (include/sched.h, R26-R28, R30)
SCHED_MODEL_NO_INTERFERENCE = 2
SCHED_MODEL_POWER_CAP = 4
SCHED_MODEL_TIME_SLICE = 8       # R30: time slicing instead of MPS (generic kernel)
UINT64_MAX = (1 << 64) - 1

EXPORTS = ["sched_create", "sched_destroy", "sched_count", "sched_workspace_size", "sched_stage",
           "sched_search", "sched_merge", "sched_unrank", "sched_rank", "sched_score", "sched_heuristic",
           "sched_strerror", "sched_version", "sched_dp_workspace_size", "sched_front_dp",
           "sched_split_workspace_size", "sched_search_splits", "sched_unrank_device",
           "sched_debug_scores32"]


class SchedError(RuntimeError):
    def __init__(self, status, what=""):
        self.status = status
        super().__init__(f"{what}: {lib().sched_strerror(status).decode()} ({status})")


class _Profile(C.Structure):
    _fields_ = [("n_workflows", C.c_int32), ("n_levels", C.c_int32),
                ("level_pct", C.POINTER(C.c_int32)), ("solo_time_s", C.POINTER(C.c_float)),
                ("solo_power_w", C.POINTER(C.c_float)), ("sm_util", C.POINTER(C.c_float)),
                ("bw_util", C.POINTER(C.c_float)), ("max_mem_mib", C.POINTER(C.c_int32)),
                ("corun_slowdown", C.POINTER(C.c_float)), ("mem_capacity_mib", C.c_int32),
                ("static_power_w", C.c_float)]


class _Query(C.Structure):
    _fields_ = [("n", C.c_int32), ("g", C.c_int32), ("max_clients", C.c_int32),
                ("level_mask", C.c_uint32), ("level_scope", C.c_int32), ("n_weights", C.c_int32),
                ("weights", C.POINTER(C.c_int32)), ("index_lo", C.c_uint64), ("index_hi", C.c_uint64),
                ("shard_rank", C.c_int32), ("shard_count", C.c_int32), ("chunk_log2", C.c_int32),
                ("want_pareto", C.c_int32), ("candidate_cap", C.c_uint32),
                ("model_flags", C.c_uint32), ("power_cap_w", C.c_float)]


class Pick(C.Structure):
    _fields_ = [("index", C.c_uint64), ("score64", C.c_double), ("x64", C.c_double),
                ("y64", C.c_double), ("makespan_s", C.c_double), ("energy_j", C.c_double),
                ("score32", C.c_float), ("x32", C.c_float), ("y32", C.c_float), ("valid", C.c_int32)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class Stats(C.Structure):
    _fields_ = [("n_configs", C.c_uint64), ("n_feasible", C.c_uint64), ("n_refined", C.c_uint64),
                ("n_candidates", C.c_uint64), ("t_seq_s", C.c_double), ("e_seq_j", C.c_double),
                ("search_ms", C.c_float), ("total_ms", C.c_float), ("kernel_path", C.c_int32),
                ("grid_ctas", C.c_int32), ("kernel_launches", C.c_int32), ("passes", C.c_int32),
                ("h2d_bytes", C.c_uint64), ("d2h_bytes", C.c_uint64), ("main_ms", C.c_float)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = None


def lib():
    """Load libsched.so (raises if the CUDA extension was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise ImportError(f"{SO_PATH} missing: run paper_conf_sc_weaverkmeh0m24_b200.build "
                              "(there is no CPU fallback)")
        L = C.CDLL(SO_PATH)
        for name in EXPORTS:
            getattr(L, name)
        L.sched_strerror.restype = C.c_char_p
        L.sched_version.restype = C.c_char_p
        for name in EXPORTS:
            if name not in ("sched_strerror", "sched_version"):
                getattr(L, name).restype = C.c_int
        _lib = L
    return _lib


def _check(st, what):
    if st != SCHED_OK:
        raise SchedError(st, what)


class DPPoint(C.Structure):
    _fields_ = [("makespan_s", C.c_double), ("energy_j", C.c_double), ("x64", C.c_double),
                ("y64", C.c_double), ("score64", C.c_double), ("n_groups", C.c_int32),
                ("group_of", C.c_int8 * 32), ("level_of", C.c_int8 * 32), ("valid", C.c_int32)]


class SplitPick(C.Structure):
    _fields_ = [("pick", Pick), ("split_rank", C.c_uint32), ("n_clients", C.c_int32),
                ("split", C.c_int32 * 32)]


@dataclasses.dataclass
class SearchResult:
    status: int
    best: list            # [W] Pick (valid=0 if none)
    pareto: list          # Pick, X descending
    stats: dict

    @property
    def best_indices(self):
        return [b.index if b.valid else None for b in self.best]

    @property
    def pareto_indices(self):
        return [p.index for p in self.pareto]


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


class Scheduler:
    """Owns a sched_handle built from a profile (host tables are copied)."""

    def __init__(self, profile):
        self._keep = [_i32(profile.level_pct), _f32(profile.solo_time_s), _f32(profile.solo_power_w),
                      _f32(profile.sm_util), _f32(profile.bw_util), _i32(profile.max_mem_mib),
                      _f32(profile.corun_slowdown)]
        k = self._keep
        P = _Profile(int(k[1].shape[0]), int(k[0].shape[0]),
                     k[0].ctypes.data_as(C.POINTER(C.c_int32)), k[1].ctypes.data_as(C.POINTER(C.c_float)),
                     k[2].ctypes.data_as(C.POINTER(C.c_float)), k[3].ctypes.data_as(C.POINTER(C.c_float)),
                     k[4].ctypes.data_as(C.POINTER(C.c_float)), k[5].ctypes.data_as(C.POINTER(C.c_int32)),
                     k[6].ctypes.data_as(C.POINTER(C.c_float)), int(profile.mem_capacity_mib),
                     float(profile.static_power_w))
        self.level_pct = [int(x) for x in k[0]]
        self._h = C.c_void_p()
        _check(lib().sched_create(C.byref(P), C.byref(self._h)), "sched_create")
        self._ws = None

    def close(self):
        if self._h:
            lib().sched_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- query marshalling --
    def cquery(self, q, shard=(0, 1), chunk_log2=24, candidate_cap=0):
        mask = 0
        for v in q.levels:
            mask |= 1 << self.level_pct.index(int(v))
        w = _i32(np.array(q.weights, dtype=np.int32).reshape(-1)) if q.weights else _i32([0, 0])
        hi = UINT64_MAX if q.index_hi is None else int(q.index_hi)
        cq = _Query(q.n, q.g, q.c, mask, q.scope, len(q.weights), w.ctypes.data_as(C.POINTER(C.c_int32)),
                    int(q.index_lo), hi, int(shard[0]), int(shard[1]), int(chunk_log2),
                    int(bool(q.want_pareto)), int(candidate_cap), int(getattr(q, "model", 0)),
                    float(getattr(q, "power_cap", 0.0)))
        cq._keep = w
        return cq

    def workspace_size(self, q, **kw) -> int:
        n = C.c_size_t()
        _check(lib().sched_workspace_size(self._h, C.byref(self.cquery(q, **kw)), C.byref(n)),
               "sched_workspace_size")
        return n.value

    def workspace(self, q, **kw):
        import torch
        n = self.workspace_size(q, **kw)
        if self._ws is None or self._ws.numel() < n:
            self._ws = torch.empty(n, dtype=torch.uint8, device="cuda")
        return self._ws

    def stage(self, q, workspace=None, stream=None, **kw):
        import torch
        ws = workspace if workspace is not None else self.workspace(q, **kw)
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        _check(lib().sched_stage(self._h, C.byref(self.cquery(q, **kw)), C.c_void_p(ws.data_ptr()),
                                 C.c_size_t(ws.numel()), C.c_void_p(st)), "sched_stage")

    def search(self, q, workspace=None, stream=None, pareto_cap=1 << 16, allow_infeasible=True,
               allow_capacity=False, **kw) -> SearchResult:
        import torch
        ws = workspace if workspace is not None else self.workspace(q, **kw)
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        nw = len(q.weights)
        best = (Pick * max(1, nw))()
        par = (Pick * max(1, pareto_cap))()
        npar = C.c_uint64()
        stats = Stats()
        rc = lib().sched_search(self._h, C.byref(self.cquery(q, **kw)), C.c_void_p(ws.data_ptr()),
                                C.c_size_t(ws.numel()), C.c_void_p(st), best, par, C.c_uint64(pareto_cap),
                                C.byref(npar), C.byref(stats))
        if rc != SCHED_OK and not (rc == SCHED_E_INFEASIBLE and allow_infeasible) and \
                not (rc == SCHED_E_CAPACITY and allow_capacity):
            raise SchedError(rc, "sched_search")
        npv = min(npar.value, pareto_cap) if q.want_pareto else 0
        return SearchResult(rc, [best[w] for w in range(nw)], [par[k] for k in range(npv)],
                            stats.as_dict())

    def dp_workspace(self, q):
        """A device workspace sized for sched_front_dp of q (caller-owned)."""
        import torch
        n = C.c_size_t()
        _check(lib().sched_dp_workspace_size(self._h, C.byref(self.cquery(q)), C.byref(n)),
               "sched_dp_workspace_size")
        return torch.empty(n.value, dtype=torch.uint8, device="cuda")

    def front_dp(self, q, workspace=None, stream=None, front_cap=4096):
        """Exact Pareto front and per-weight optimum of the whole space by the
        device subset DP (sched_front_dp).  Returns (status, best[W], front,
        stats); points carry one witness configuration (group_of, level_of)."""
        import torch
        n = C.c_size_t()
        cq = self.cquery(q)
        _check(lib().sched_dp_workspace_size(self._h, C.byref(cq), C.byref(n)), "sched_dp_workspace_size")
        ws = workspace if workspace is not None else torch.empty(n.value, dtype=torch.uint8, device="cuda")
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        nw = len(q.weights)
        best = (DPPoint * max(1, nw))()
        front = (DPPoint * front_cap)()
        nf = C.c_uint64()
        stats = Stats()
        rc = lib().sched_front_dp(self._h, C.byref(cq), C.c_void_p(ws.data_ptr()), C.c_size_t(ws.numel()),
                                  C.c_void_p(st), best, front, C.c_uint64(front_cap), C.byref(nf),
                                  C.byref(stats))
        if rc not in (SCHED_OK, SCHED_E_INFEASIBLE):
            raise SchedError(rc, "sched_front_dp")
        return rc, [best[w] for w in range(nw)], [front[i] for i in range(min(nf.value, front_cap))], \
            stats.as_dict()

    def search_splits(self, q, tasks, max_split=None, stream=None, pareto_cap=4096):
        """Scheduling-configuration search (sched_search_splits; SURVEY 8(f) N3,
        DESIGN.md R29): every split of workflow i's tasks[i] tasks into
        concurrent clients x every configuration of the expanded queue.
        Returns (status, best[W], pareto, stats, n_splits); picks are
        SplitPick (pick, split_rank, n_clients, split[])."""
        import torch
        t = _i32(tasks)
        ms = None if max_split is None else _i32(max_split)
        tp = t.ctypes.data_as(C.POINTER(C.c_int32))
        mp = None if ms is None else ms.ctypes.data_as(C.POINTER(C.c_int32))
        cq = self.cquery(q)
        n = C.c_size_t()
        ns = C.c_uint32()
        _check(lib().sched_split_workspace_size(self._h, C.byref(cq), tp, mp, C.byref(n), C.byref(ns)),
               "sched_split_workspace_size")
        if self._ws is None or self._ws.numel() < n.value:
            self._ws = torch.empty(n.value, dtype=torch.uint8, device="cuda")
        ws = self._ws
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        nw = len(q.weights)
        best = (SplitPick * max(1, nw))()
        par = (SplitPick * max(1, pareto_cap))()
        npar = C.c_uint64()
        stats = Stats()
        rc = lib().sched_search_splits(self._h, C.byref(cq), tp, mp, C.c_void_p(ws.data_ptr()),
                                       C.c_size_t(ws.numel()), C.c_void_p(st), best, par,
                                       C.c_uint64(pareto_cap), C.byref(npar), C.byref(stats))
        if rc not in (SCHED_OK, SCHED_E_INFEASIBLE):
            raise SchedError(rc, "sched_search_splits")
        npv = min(npar.value, pareto_cap) if q.want_pareto else 0
        return rc, [best[w] for w in range(nw)], [par[k] for k in range(npv)], stats.as_dict(), ns.value

    def heuristic(self, q, priority="throughput", w=0):
        """The paper's rule-based scheduler (criteria 1-4).
        Returns (group_of, level_of, index, Pick)."""
        a = (C.c_int8 * 32)()
        lv = (C.c_int8 * 32)()
        idx = C.c_uint64()
        out = Pick()
        pr = {"throughput": 0, "energy": 1}[priority]
        _check(lib().sched_heuristic(self._h, C.byref(self.cquery(q)), pr, w, a, lv, C.byref(idx), C.byref(out)),
               "sched_heuristic")
        return [a[i] for i in range(q.n)], [lv[i] for i in range(q.n)], idx.value, out

    def unrank_device(self, q, indices, advance=0, workspace=None, stream=None):
        """Device unrank (+ `advance` successor steps) of a uint64 tensor of
        indices (sched_unrank_device).  Returns (group_of, level_of) int8
        device tensors [n][q.n]; rows of out-of-range indices have
        group_of[:, 0] = -1."""
        import torch
        idx = indices.to(device="cuda", dtype=torch.int64).contiguous()
        n = idx.numel()
        g = torch.empty((n, q.n), dtype=torch.int8, device="cuda")
        lv = torch.empty((n, q.n), dtype=torch.int8, device="cuda")
        ws = workspace if workspace is not None else self.workspace(q)
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        _check(lib().sched_unrank_device(self._h, C.byref(self.cquery(q)), C.c_void_p(idx.data_ptr()),
                                         C.c_uint64(n), C.c_uint64(advance), C.c_void_p(g.data_ptr()),
                                         C.c_void_p(lv.data_ptr()), C.c_void_p(ws.data_ptr()),
                                         C.c_size_t(ws.numel()), C.c_void_p(st)), "sched_unrank_device")
        return g, lv

    def debug_scores32(self, q, stream=None):
        """fp32 hot-loop (T/T_seq, E/E_seq) of every configuration of q's
        window on the tile kernel (sched_debug_scores32); NaN rows where the
        partition is memory-infeasible.  Returns a float32 device tensor [n, 2]."""
        import torch
        n = int(q.index_hi) - int(q.index_lo)
        out = torch.full((n, 2), float("nan"), dtype=torch.float32, device="cuda")
        qq = dataclasses.replace(q, weights=((1, 1),), want_pareto=False)
        ws = self.workspace(qq)
        st = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        _check(lib().sched_debug_scores32(self._h, C.byref(self.cquery(qq)), C.c_void_p(ws.data_ptr()),
                                          C.c_size_t(ws.numel()), C.c_void_p(st), C.c_void_p(out.data_ptr())),
               "sched_debug_scores32")
        return out

    def score(self, q, index, w=0) -> Pick:
        out = Pick()
        _check(lib().sched_score(self._h, C.byref(self.cquery(q)), C.c_uint64(index), w, C.byref(out)),
               "sched_score")
        return out


def _shape_query(q):
    mask = (1 << len(q.levels)) - 1   # shape-only calls: only L = popcount matters
    cq = _Query(q.n, q.g, q.c, mask, q.scope, 0, None, 0, UINT64_MAX, 0, 1, 22, 0, 0, 0, 0.0)
    return cq


def count(q) -> int:
    v = C.c_uint64()
    _check(lib().sched_count(C.byref(_shape_query(q)), C.byref(v)), "sched_count")
    return v.value


def unrank(q, index):
    a = (C.c_int8 * 32)()
    lv = (C.c_int8 * 32)()
    _check(lib().sched_unrank(C.byref(_shape_query(q)), C.c_uint64(index), a, lv), "sched_unrank")
    return [a[i] for i in range(q.n)], [lv[i] for i in range(q.n)]


def rank(q, group_of, level_of) -> int:
    a = (C.c_int8 * 32)(*group_of)
    lv = (C.c_int8 * 32)(*level_of)
    v = C.c_uint64()
    _check(lib().sched_rank(C.byref(_shape_query(q)), a, lv, C.byref(v)), "sched_rank")
    return v.value


def merge(rank_best, rank_pareto, n_weights, pareto_cap=1 << 16):
    """rank_best: list (per rank) of W Picks; rank_pareto: list (per rank) of Pick lists."""
    R = len(rank_best)
    rb = (Pick * max(1, R * n_weights))()
    for r in range(R):
        for w in range(n_weights):
            rb[r * n_weights + w] = rank_best[r][w]
    allp = [p for lst in rank_pareto for p in lst]
    rp = (Pick * max(1, len(allp)))(*allp)
    rn = (C.c_uint64 * R)(*[len(x) for x in rank_pareto])
    best = (Pick * max(1, n_weights))()
    par = (Pick * max(1, pareto_cap))()
    npar = C.c_uint64()
    _check(lib().sched_merge(R, n_weights, rb, rp, rn, best, par, C.c_uint64(pareto_cap), C.byref(npar)),
           "sched_merge")
    return [best[w] for w in range(n_weights)], [par[k] for k in range(npar.value)]


def version() -> str:
    return lib().sched_version().decode()
