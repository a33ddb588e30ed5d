"""Time bench-shaped searches (one 1/64 cyclic chunk slice of a workload,
2^24-index chunks) under several weight sets / kernels:
  python tools/time_slices.py c4 [--sets c4,c1_set,c5_sweep,eight] [--reps 3] [--sigma 5]
One JSON line per (set, rep): device search_ms, configs/s, kernel path."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config, Query  # noqa: E402

SETS = {
    "c4": None,
    "c1_set": ((1, 0), (0, 1), (1, 1), (2, 1)),
    "c5_sweep": ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1)),
    "eight": ((1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (4, 4)),
    "pareto": (),
    "w11": ((1, 1),),
    "w10": ((1, 0),),
    "w10_01": ((1, 0), (0, 1)),
    "w11_21_12": ((1, 1), (2, 1), (1, 2)),
}

ap = argparse.ArgumentParser()
ap.add_argument("name", nargs="?", default="c4")
ap.add_argument("--sets", default="c4,c1_set,c5_sweep")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--sigma", type=int, default=5)
ap.add_argument("--slices", type=int, default=64)
ap.add_argument("--scope", type=int, default=None)
ap.add_argument("--levels", default=None, help="comma-separated MPS levels, e.g. 50,75,100")
a = ap.parse_args()
prof, q = config(a.name)
if a.scope is not None or a.levels:
    lv = tuple(int(x) for x in a.levels.split(",")) if a.levels else q.levels
    q = Query(q.n, q.g, q.c, lv, q.scope if a.scope is None else a.scope, q.weights, q.want_pareto)
sch = S.Scheduler(prof)
for s in a.sets.split(","):
    qs = q if SETS[s] is None else Query(q.n, q.g, q.c, q.levels, q.scope, SETS[s], q.want_pareto)
    for r in range(a.reps):
        res = sch.search(qs, shard=(a.sigma, a.slices), chunk_log2=24, allow_capacity=True)
        st = res.stats
        print(json.dumps({"workload": a.name, "set": s, "rep": r, "path": st["kernel_path"],
                          "search_ms": st["search_ms"], "configs": st["n_configs"],
                          "configs_per_s": st["n_configs"] / (st["search_ms"] / 1e3),
                          "refined": st["n_refined"], "cand": st["n_candidates"], "status": res.status,
                          "passes": st["passes"], "launches": st["kernel_launches"], "total_ms": st["total_ms"]}),
              flush=True)
