"""Literal per-client c4 (4.05e19 configurations) through sched_front_dp:
python tools/dp_c4client.py [scope]  -> one JSON line (device ms, front, best)."""
import dataclasses
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config, PER_CLIENT, PER_GPU  # noqa: E402

prof, q = config(sys.argv[1] if len(sys.argv) > 1 and sys.argv[1].startswith("c") else "c4")
scope = PER_GPU if "gpu" in sys.argv else PER_CLIENT
q = dataclasses.replace(q, scope=scope)
sch = S.Scheduler(prof)
t0 = time.perf_counter()
rc, best, front, st = sch.front_dp(q)
dt = time.perf_counter() - t0
print(json.dumps({"scope": "per_client" if scope == PER_CLIENT else "per_gpu", "status": rc, "wall_s": dt,
                  "device_ms": st["search_ms"], "front": [(p.makespan_s, p.energy_j) for p in front],
                  "best": [b.score64 for b in best], "launches": st["kernel_launches"]}))
