"""Time-to-optimal by the subset DP, cold and warm, in a fresh process:
  python tools/dp_cold.py [c4] [--after-search]
Prints one JSON line per call (wall around the C-ABI call, device ms)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

name = next((a for a in sys.argv[1:] if not a.startswith("--")), "c4")
prof, q = config(name)
torch.cuda.init()
torch.empty(1, device="cuda")
sch = S.Scheduler(prof)
if "--after-search" in sys.argv:
    sch.search(q.with_range(0, 1 << 20))
ws = None
for i in range(6):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    rc, best, front, st = sch.front_dp(q, workspace=ws)
    torch.cuda.synchronize()
    print(json.dumps({"call": i, "wall_ms": (time.perf_counter() - t0) * 1e3, "device_ms": st["total_ms"],
                      "module_loading": os.environ.get("CUDA_MODULE_LOADING", "default"),
                      "front": len(front), "best": [b.score64 for b in best]}), flush=True)
    if ws is None:
        ws = sch.dp_workspace(q)
