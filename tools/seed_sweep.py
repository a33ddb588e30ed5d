"""Seed-pass size sweep: c4 bench-step searches at R = 1 and R = 8 shares with
SCHED_SEED_UNITS_PER_SM:SCHED_SEED_UNIT_LOG2 = v (child process per value); device ms of the seed
pass is total search_ms minus the main pass (reported by the library)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, json
sys.path.insert(0, "%s")
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config
prof, q = config("c4")
sch = S.Scheduler(prof); ws = sch.workspace(q); sch.stage(q, workspace=ws)
out = {}
for R in (1, 8):
    sch.search(q, workspace=ws, shard=(0, 64 * R), chunk_log2=22)
    ms = []
    for s in range(3):
        r = sch.search(q, workspace=ws, shard=(s * R, 64 * R), chunk_log2=22)
        ms.append(r.stats["search_ms"])
        cand = r.stats["n_candidates"]; ref = r.stats["n_refined"]
    out[R] = (sum(ms) / 3, cand, ref)
print(json.dumps(out))
''' % ROOT
for v in sys.argv[1:] or ["64:12", "256:10"]:
    per_sm, ul = v.split(":")
    env = dict(os.environ, SCHED_SEED_UNITS_PER_SM=per_sm, SCHED_SEED_UNIT_LOG2=ul)
    r = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True)
    print(v, r.stdout.strip() or r.stderr[-500:], flush=True)
