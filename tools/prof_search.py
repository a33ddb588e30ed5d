"""One search through the C ABI, for ncu captures:
  python tools/prof_search.py c4 [lo n] [--scope 0|1] [--shard r R] [--weights 1,1:2,1]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config, Query  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("name", nargs="?", default="c4")
ap.add_argument("lo", nargs="?", type=int)
ap.add_argument("n", nargs="?", type=int)
ap.add_argument("--scope", type=int)
ap.add_argument("--shard", type=int, nargs=2)
ap.add_argument("--weights")
a = ap.parse_args()
prof, q = config(a.name)
if a.scope is not None or a.weights:
    ws = q.weights if not a.weights else tuple(tuple(int(x) for x in w.split(",")) for w in a.weights.split(":"))
    q = Query(q.n, q.g, q.c, q.levels, q.scope if a.scope is None else a.scope, ws, q.want_pareto)
if a.lo is not None:
    q = q.with_range(a.lo, a.lo + a.n)
sch = S.Scheduler(prof)
kw = {"shard": tuple(a.shard), "chunk_log2": 24} if a.shard else {}
r = sch.search(q, **kw)
print(a.name, r.stats, r.best_indices, len(r.pareto))
