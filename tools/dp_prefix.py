"""Per-client subset-DP front of the c4 profile's first n workflows (the O4
golden sizes): python tools/dp_prefix.py 13 -> one JSON line.  Needs a GPU."""
import dataclasses
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config, PER_CLIENT  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 13
prof, q = config("c4")
q = dataclasses.replace(q, n=n, scope=PER_CLIENT)
rc, best, front, st = S.Scheduler(prof.subset(n)).front_dp(q)
print(json.dumps({"n": n, "status": rc, "device_ms": st["total_ms"], "front": len(front)}))
