"""Optimality gap of the paper's rule-based scheduler (PAPER.md L89-L92,
sched_heuristic) on the five BASELINE workloads: its
throughput X and energy efficiency Y (throughput priority: <= 2 clients per
GPU; energy priority: up to C) against the exact optima X* = T_seq / min T
and Y* = E_seq / min E over the exact Pareto front (device subset DP for
c1-c4, the committed O3 certificate for c5).  Needs a GPU.
  python tools/heuristic_gap.py > profiles/r01_heuristic_gap.md"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

print("| cfg | X* | Y* | heuristic, throughput priority: X, Y | heuristic, energy priority: X, Y |")
print("|---|---|---|---|---|")
for name in ("c1", "c2", "c3", "c4", "c5"):
    prof, q = config(name)
    sch = S.Scheduler(prof)
    if name == "c5":
        g = json.load(open(os.path.join(ROOT, "tests", "golden", "c5_certificate.json")))
        front = [(float.fromhex(t), float.fromhex(e)) for t, e in g["front_T_E"]]
        ts, es = float.fromhex(g["tseq"]), float.fromhex(g["eseq"])
    else:
        rc, best, fr, st = sch.front_dp(q)
        front = [(p.makespan_s, p.energy_j) for p in fr]
        ts, es = st["t_seq_s"], st["e_seq_j"]
    xs = ts / min(t for t, _ in front)
    ys = es / min(e for _, e in front)
    cells = []
    for pr in ("throughput", "energy"):
        try:
            a, lv, idx, pick = sch.heuristic(q, pr, 0)
            cells.append(f"{pick.x64:.4f} ({pick.x64 / xs:.1%}), {pick.y64:.4f} ({pick.y64 / ys:.1%})"
                         if pick.valid else "infeasible (memory)")
        except S.SchedError as e:
            cells.append(f"no placement ({e.status})")
    print(f"| {name} | {xs:.4f} | {ys:.4f} | {cells[0]} | {cells[1]} |", flush=True)
