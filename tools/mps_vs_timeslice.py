"""MPS co-scheduling vs time slicing (PAPER.md L33 time slicing; L140 Fig. 2
"MPS vs time-slicing"; readings R10 / R30) on the five BASELINE workloads:
the exact optimum throughput X* and energy efficiency Y* of the whole space
under the canonical MPS model and under SCHED_MODEL_TIME_SLICE, each by one
exhaustive sched_search per weight ((1,0), then (0,1); no Pareto set), with the
device search time.  Needs a GPU.
  python tools/mps_vs_timeslice.py > profiles/r01_mps_vs_timeslice.md"""
import dataclasses
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

TIME_SLICE = S.sched.SCHED_MODEL_TIME_SLICE
print("# MPS vs time slicing: exact optima over the whole space (tools/mps_vs_timeslice.py, one B200)\n")
print("X* = T_seq / min T, Y* = E_seq / min E over every configuration; both models use the same profile, space "
      "and sequential baseline.  Time slicing (R30): the clients of a GPU run one after another at their solo "
      "profile, so its throughput optimum is a pure load balancing (P||Cmax) of the solo times; MPS can "
      "overlap them.\n")
print("| cfg | configurations | MPS: X*, Y* (search ms, path) | time slicing: X*, Y* (search ms, path) |")
print("|---|---|---|---|")
for name in ("c1", "c2", "c3", "c4", "c5"):
    prof, q = config(name)
    sch = S.Scheduler(prof)
    cells = []
    for model in (0, TIME_SLICE):
        picks, ms, paths = [], 0.0, set()
        for w in ((1, 0), (0, 1)):   # one weight per search: single-weight tile instantiations
            qm = dataclasses.replace(q, model=model, weights=(w,), want_pareto=False)
            t0 = time.time()
            r = sch.search(qm)
            print(f"  {name} model={model} w={w} wall {time.time() - t0:.2f} s", file=sys.stderr, flush=True)
            picks.append(r.best[0])
            ms += r.stats["search_ms"]
            paths.add(r.stats["kernel_path"])
        bx, by = picks
        cells.append(f"{bx.x64:.4f}, {by.y64:.4f} ({ms:.1f} ms, path {'/'.join(map(str, sorted(paths)))})"
                     if bx.valid else "infeasible")
    print(f"| {name} | {S.count(q):,} | {cells[0]} | {cells[1]} |", flush=True)
