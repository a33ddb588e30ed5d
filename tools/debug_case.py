"""Debug one search: python tools/debug_case.py  (prints stats per kernel)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import make_profile, Query, PER_CLIENT  # noqa: E402

LV = (25, 50, 75, 100)
prof = make_profile(8, levels=LV, seed=606)
q = Query(8, 8, 3, LV, PER_CLIENT, ((1, 1), (2, 1), (1, 0), (0, 1)), True)
ref = oracle.search_parallel(prof, q)
print("oracle pareto", len(ref["pareto"]), "best", [b[0] for b in ref["best"]], flush=True)
for kern in ("ctile", "ctile2", "generic"):
    os.environ["SCHED_KERNEL"] = kern
    r = S.Scheduler(prof).search(q, allow_capacity=True)
    print(kern, "status", r.status, {k: r.stats[k] for k in ("kernel_path", "n_configs", "n_feasible", "n_refined",
                                                           "n_candidates", "passes")},
          "npareto", len(r.pareto), "best", [b.index for b in r.best], flush=True)
    print("  pareto equal:", [(p.index, p.makespan_s, p.energy_j) for p in r.pareto] == ref["pareto"])
