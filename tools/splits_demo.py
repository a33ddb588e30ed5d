"""Scheduling-configuration search (sched_search_splits) on
the paper's cardinality experiment shape: LAMMPS and
AthenaPK workflows of 4 tasks each on the paper's 2 GPUs (L63), every split
'4-1', '2-2', '1-4' per workflow x every co-schedule of the resulting
clients.  Needs a GPU.  python tools/splits_demo.py -> JSON lines."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import make_profile, Query, PER_GPU  # noqa: E402

LAMMPS_4X, ATHENAPK_4X = 10, 1
for arch in ([LAMMPS_4X, ATHENAPK_4X], [LAMMPS_4X, ATHENAPK_4X, LAMMPS_4X, ATHENAPK_4X]):
    n = len(arch)
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=7, archetypes=arch)
    q = Query(n, 2, 16, (25, 50, 75, 100), PER_GPU, ((1, 0), (0, 1), (1, 1)), True)
    sch = S.Scheduler(prof)
    t0 = time.perf_counter()
    rc, best, par, st, ns = sch.search_splits(q, [4] * n)
    dt = time.perf_counter() - t0
    print(json.dumps({"workflows": [prof.names[i] for i in range(n)], "tasks": [4] * n, "gpus": 2,
                      "splits": ns, "configs": st["n_configs"], "wall_s": dt, "device_ms": st["total_ms"],
                      "best": [{"weight": list(w), "X": b.pick.x64, "Y": b.pick.y64, "split": list(b.split)[:n],
                                "clients": b.n_clients} for w, b in zip(q.weights, best)],
                      "pareto": len(par)}), flush=True)
