set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
python - <<'PY'
import time, torch
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config
for name, rng in [("c2",None),("c3",None),("c4",(10**14, 10**14 + 2**36)),("c4",None),("c5",(3*10**11, 3*10**11+2**33))]:
    prof,q = config(name)
    sch = S.Scheduler(prof)
    if rng: q = q.with_range(*rng)
    if name == "c4" and rng is None:
        t=time.time(); r = sch.search(q); dt=time.time()-t
    else:
        r = sch.search(q)
        t=time.time(); r = sch.search(q); dt=time.time()-t
    st = r.stats
    print(name, rng, "configs", st["n_configs"], "feas", st["n_feasible"], "path", st["kernel_path"], "grid", st["grid_ctas"], "search_ms", st["search_ms"], "wall", dt,
          "cfg/s %.4g" % (st["n_configs"]/(st["search_ms"]/1e3)), "refined", st["n_refined"], "cand", st["n_candidates"], "pareto", len(r.pareto), "best", r.best_indices, [b.score64 for b in r.best], flush=True)
PY
