"""One small search through every kernel path, for compute-sanitizer
(SURVEY 5 "race detection / sanitizers"): generic, tile, PER_CLIENT tile,
suffix, pair (DFS) kernels, the group table, the finalize kernels, the
subset-DP front and a split search.  Each result is checked against the
oracle so a sanitizer run also shows that the instrumented run is correct.
  compute-sanitizer --tool memcheck  python tools/sanitize_paths.py
  compute-sanitizer --tool racecheck python tools/sanitize_paths.py
  compute-sanitizer --tool synccheck python tools/sanitize_paths.py
(tools/gpu_scripts/sanitize.sh runs all three; summary in profiles/r01_sanitizer.md)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402  (test infrastructure: checking the instrumented runs)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import make_profile, Query, PER_CLIENT, PER_GPU  # noqa: E402

W = ((1, 1), (2, 1))
SWEEP = ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1))
CASES = [  # name, SCHED_KERNEL, expected path, n, g, c, levels, scope, weights, seed
    ("generic", "generic", 0, 6, 3, 6, (50, 100), PER_CLIENT, W, 1),
    ("tile", "tile", 1, 9, 6, 3, (25, 50, 75, 100), PER_GPU, W, 2),
    ("ctile", "ctile", 5, 7, 3, 7, (25, 50, 75, 100), PER_CLIENT, W, 3),
    ("sfx", "sfx", 3, 10, 5, 3, (100,), PER_GPU, SWEEP, 4),
    ("dfs", "dfs", 2, 10, 5, 3, (100,), PER_GPU, SWEEP, 4),
    ("ctile2", "ctile2", 6, 7, 4, 3, (25, 50, 75, 100), PER_CLIENT, W, 7),        # round 2: group-table PER_CLIENT
    ("tile_rt", "tile", 1, 9, 6, 3, (25, 50, 75, 100), PER_GPU, ((1, 2), (3, 1), (1, 0)), 8),   # run-time weights
    ("tile_rtn", "tile", 1, 9, 6, 3, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1), (1, 2)), 9),  # run-time, b >= 1
    ("sfx_c", "sfx", 3, 11, 6, 3, (100,), PER_GPU, ((1, 1), (2, 1)), 10),     # pair tiles, capped groups
]


def same(res, ref):
    got = [b.index if b.valid else None for b in res.best]
    want = [b[0] if b else None for b in ref["best"]]
    assert got == want, (got, want)
    assert [(p.index, p.makespan_s, p.energy_j) for p in res.pareto] == [tuple(x) for x in ref["pareto"]]


ONLY = set(sys.argv[1:])   # optional: run only these cases (names as below, plus front_dp, splits)
for name, kern, path, n, g, c, levels, scope, weights, seed in CASES:
    if ONLY and name not in ONLY:
        continue
    os.environ["SCHED_KERNEL"] = kern
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed, g=g, c=c)
    q = Query(n, g, c, levels, scope, weights, True)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == path, (name, res.stats["kernel_path"])
    same(res, oracle.search(prof, q))
    print(f"{name}: ok ({S.count(q)} configurations)", flush=True)
os.environ.pop("SCHED_KERNEL", None)

if not ONLY or "front_dp" in ONLY:
    prof = make_profile(7, levels=(25, 50, 75, 100), seed=5)
    q = Query(7, 3, 7, (50, 100), PER_CLIENT, W, True)
    rc, best, front, st = S.Scheduler(prof).front_dp(q)
    ref = oracle.search(prof, q)
    assert sorted((p.makespan_s, p.energy_j) for p in front) == sorted((t, e) for _, t, e in ref["pareto"])
    print(f"front_dp: ok ({len(front)} points)", flush=True)

if not ONLY or "unrank_device" in ONLY:
    import torch
    prof = make_profile(8, levels=(25, 50, 75, 100), seed=9)
    q = Query(8, 4, 8, (25, 50, 75, 100), PER_GPU, W, True)
    sch = S.Scheduler(prof)
    idx = torch.arange(0, S.count(q), 97, dtype=torch.int64)
    g, lv = sch.unrank_device(q, idx, advance=3)
    g = g.cpu().tolist()
    for t in range(0, len(g), 50):
        i = int(idx[t]) + 3
        if i < S.count(q):
            assert g[t] == oracle.config(q, i)[0]
    print("unrank_device: ok", flush=True)

if not ONLY or "scores32" in ONLY:
    import math
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=10)
    q = Query(9, 6, 3, (25, 50, 75, 100), PER_GPU, ((1, 1),), False, 1000, 21000)
    out = S.Scheduler(prof).debug_scores32(q).cpu().tolist()
    T, E = oracle.score_window(prof, q)
    ts, es = oracle.constants(prof, q)
    for k in range(0, 20000, 37):
        if not math.isnan(T[k]):
            assert abs(out[k][0] / (T[k] / ts) - 1) <= 1e-5
    print("debug_scores32: ok", flush=True)

if not ONLY or "splits" in ONLY:
    prof = make_profile(3, levels=(50, 100), seed=6)
    q = Query(3, 2, 3, (50, 100), PER_GPU, W, True)
    rc, sbest, spar, sst, nsplit = S.Scheduler(prof).search_splits(q, [2, 2, 1])
    assert rc == S.sched.SCHED_OK and nsplit == 4
    print(f"search_splits: ok ({nsplit} splits)", flush=True)
print("ALL PATHS OK")
