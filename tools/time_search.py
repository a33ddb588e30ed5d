"""Time searches through the C ABI: python tools/time_search.py c5 [lo n] [--reps K].
Prints one JSON line per rep (device search_ms, wall, stats, picks)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

args = [a for a in sys.argv[1:] if not a.startswith("--")]
reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 1
if "--reps" in sys.argv:
    args = [a for a in args if a != str(reps)]
name = args[0] if args else "c5"
prof, q = config(name)
if len(args) >= 3:
    lo, n = int(args[1]), int(args[2])
    q = q.with_range(lo, lo + n)
sch = S.Scheduler(prof)
for _ in range(reps):
    t0 = time.perf_counter()
    r = sch.search(q, allow_capacity=True)
    dt = time.perf_counter() - t0
    st = r.stats
    print(json.dumps({"name": name, "kernel": os.environ.get("SCHED_KERNEL", "auto"), "wall_s": dt,
                      "search_ms": st["search_ms"], "configs": st["n_configs"],
                      "configs_per_s": st["n_configs"] / (st["search_ms"] / 1e3),
                      "path": st["kernel_path"], "status": r.status, "passes": st["passes"], "cand": st["n_candidates"],
                      "refined": st["n_refined"], "feasible": st["n_feasible"],
                      "best": [(b.index, b.score64) for b in r.best],
                      "pareto": [(p.index, p.makespan_s, p.energy_j) for p in r.pareto]}))
