timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
python - <<'PY'
import time
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config
for name, rng in [("c3",None),("c4",(10**14, 10**14 + 2**36)),("c4",(3*10**13, 3*10**13 + 2**38))]:
    prof,q = config(name)
    sch = S.Scheduler(prof)
    if rng: q = q.with_range(*rng)
    r = sch.search(q)
    r = sch.search(q)
    st = r.stats
    print(name, rng, "configs", st["n_configs"], "path", st["kernel_path"], "grid", st["grid_ctas"], "search_ms %.1f" % st["search_ms"],
          "cfg/s %.4g" % (st["n_configs"]/(st["search_ms"]/1e3)), "refined", st["n_refined"], "cand", st["n_candidates"], "pareto", len(r.pareto), "best", r.best_indices, flush=True)
PY
python bench.py --steps 3 --warmup 3 --no-cpu-baseline
