"""One search through the C ABI, for ncu captures: python tools/prof_search.py c4 [lo] [n]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c4"
prof, q = config(name)
if len(sys.argv) > 3:
    lo, n = int(sys.argv[2]), int(sys.argv[3])
    q = q.with_range(lo, lo + n)
sch = S.Scheduler(prof)
r = sch.search(q)
print(name, r.stats, r.best_indices, len(r.pareto))
