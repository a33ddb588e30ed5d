"""Load balance of the multi-GPU split measured on ONE B200:
the bench step (one 1/64 cyclic chunk slice of c4) is split over R ranks
exactly as bench.py does (shard = slice * R + rank of 64 * R), and each
rank's share is searched in turn on the one GPU.  Reports, per R, the
per-rank device search times and the strong-scaling efficiency the split
allows, T(1) / (R * max_r T_r) -- the ceiling of the driver's 1 -> R GPU
scaling (the NCCL exchange of a few KB per step is not included; the box
has one GPU, so it cannot be measured here).
  python tools/shard_balance.py > profiles/r02_shard_balance.md"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

SLICES, CHUNK_LOG2 = 64, 24   # as bench.py
prof, q = config("c4")
sch = S.Scheduler(prof)
ws = sch.workspace(q)
sch.stage(q, workspace=ws)
STEPS = (0, 1, 2)
for s in STEPS:   # warm-up
    sch.search(q, workspace=ws, shard=(s, SLICES), chunk_log2=CHUNK_LOG2)

print("# Multi-GPU split balance (tools/shard_balance.py, one B200, c4 bench steps 0-2)\n")
print("| R | per-rank device ms (mean over 3 steps) | max / mean | configs per rank (max / min) "
      "| split-limited efficiency T1 / (R max T_r) |")
print("|---|---|---|---|---|")
t1 = None
for R in (1, 2, 4, 8):
    per = []
    cfg = []
    for r in range(R):
        ms, n = 0.0, 0
        for s in STEPS:
            res = sch.search(q, workspace=ws, shard=(s * R + r, SLICES * R), chunk_log2=CHUNK_LOG2)
            ms += res.stats["search_ms"]
            n += res.stats["n_configs"]
        per.append(ms / len(STEPS))
        cfg.append(n)
    mx, mean = max(per), sum(per) / R
    if R == 1:
        t1 = per[0]
    eff = t1 / (R * mx)
    print(f"| {R} | {', '.join(f'{x:.1f}' for x in per)} | {mx / mean:.3f} | {max(cfg) / min(cfg):.4f} "
          f"| {eff:.3f} |", flush=True)
