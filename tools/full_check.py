"""Exhaustive searches of whole spaces on the GPU compared with the committed
exact certificates (tests/golden/<name>_certificate.json, written by
oracle/make_certificates.py): best fp64 score per weight and the Pareto
front's (T, E) values bitwise.  c4 runs as 64 cyclic chunk slices merged with
sched_merge (the bench's --full path).
  python tools/full_check.py c3 c5 c4
One JSON line per space."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402


def hx(x):
    return float.hex(float(x))


for name in sys.argv[1:] or ["c3", "c5", "c4"]:
    cert = json.load(open(os.path.join(ROOT, "tests", "golden", f"{name}_certificate.json")))
    prof, q = config(name)
    sch = S.Scheduler(prof)
    t0 = time.perf_counter()
    if name == "c4":
        bests, pars, n, ms = [], [], 0, 0.0
        for sigma in range(64):
            r = sch.search(q, shard=(sigma, 64), chunk_log2=24)
            bests.append(r.best)
            pars.append(r.pareto)
            n += r.stats["n_configs"]
            ms += r.stats["search_ms"]
        best, front = S.merge(bests, pars, len(q.weights))
    else:
        r = sch.search(q)
        best, front, n, ms = r.best, r.pareto, r.stats["n_configs"], r.stats["search_ms"]
    wall = time.perf_counter() - t0
    got_best = [hx(b.score64) for b in best]
    got_front = sorted([hx(p.makespan_s), hx(p.energy_j)] for p in front)
    want_front = sorted([t, e] for t, e in cert["front_T_E"])
    ok = got_best == cert["best_score64"] and got_front == want_front
    print(json.dumps({"space": name, "configs": n, "count": S.count(q), "search_ms": ms, "wall_s": wall,
                      "best_equal": got_best == cert["best_score64"], "front_equal": got_front == want_front,
                      "front_points": len(front), "ok": ok and n == S.count(q)}), flush=True)
