"""c4 bench-step device time vs chunk size (2^chunk_log2 indices; the tile
kernel's units are capped at one chunk): R = 1 and R = 8 shares."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_weaverkmeh0m24_b200 as S  # noqa: E402
from synth import config  # noqa: E402

prof, q = config("c4")
sch = S.Scheduler(prof)
ws = sch.workspace(q)
sch.stage(q, workspace=ws)
for cl in [int(x) for x in sys.argv[1:]] or [22, 23, 24]:
    for R in (1, 8):
        sch.search(q, workspace=ws, shard=(0, 64 * R), chunk_log2=cl)
        ms, n = [], 0
        for s in range(3):
            r = sch.search(q, workspace=ws, shard=(s * R, 64 * R), chunk_log2=cl)
            ms.append(r.stats["search_ms"])
            n += r.stats["n_configs"]
        print(f"chunk 2^{cl} R={R}: {sum(ms) / 3:.2f} ms/step  {n / (sum(ms) / 1e3):.4e} configs/s  "
              f"cand {r.stats['n_candidates']}", flush=True)
