"""One bench-step search at R ranks (shard 0 of 64*R), for ncu launch lists
of the per-search fixed costs (tools/shard_balance.py)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

R = int(sys.argv[1]) if len(sys.argv) > 1 else 8
prof, q = config("c4")
sch = S.Scheduler(prof)
ws = sch.workspace(q)
sch.stage(q, workspace=ws)
res = sch.search(q, workspace=ws, shard=(0, 64 * R), chunk_log2=22)
print(res.stats)
