echo "start $(date +%s)"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
echo "tests done $(date +%s)"
timeout 600 python - <<'PY'
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config
for name, rng in [("c3",None),("c4",(3*10**13, 3*10**13 + 2**38)),("c5",(3*10**11, 3*10**11+2**33)),("c5",None)]:
    prof,q = config(name)
    sch = S.Scheduler(prof)
    if rng: q = q.with_range(*rng)
    r = sch.search(q); r = sch.search(q)
    st = r.stats
    print(name, rng, "configs", st["n_configs"], "path", st["kernel_path"], "grid", st["grid_ctas"], "search_ms %.1f" % st["search_ms"],
          "cfg/s %.4g" % (st["n_configs"]/(st["search_ms"]/1e3)), "refined", st["n_refined"], "cand", st["n_candidates"], "passes", st["passes"], "pareto", len(r.pareto), "best", r.best_indices, [b.score64 for b in r.best], flush=True)
PY
echo "perf done $(date +%s)"
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline
