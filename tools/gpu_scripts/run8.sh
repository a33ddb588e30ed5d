timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "partition or c5 or small or edge" 2>&1 | tail -3
python - <<'PY'
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config
for name, rng in [("c5",(3*10**11, 3*10**11+2**33)),("c5",None)]:
    prof,q = config(name)
    sch = S.Scheduler(prof)
    if rng: q = q.with_range(*rng)
    r = sch.search(q); r = sch.search(q)
    st = r.stats
    print(name, rng, "configs", st["n_configs"], "path", st["kernel_path"], "grid", st["grid_ctas"], "search_ms %.1f" % st["search_ms"],
          "cfg/s %.4g" % (st["n_configs"]/(st["search_ms"]/1e3)), "refined", st["n_refined"], "cand", st["n_candidates"], "passes", st["passes"], "pareto", len(r.pareto), "best", r.best_indices, [b.score64 for b in r.best], flush=True)
PY
ncu --set full --clock-control none --import-source on -k regex:k_dfs -c 1 -o gpurun_out/prof_pair_c5 python tools/prof_search.py c5 300000000000 8589934592 > gpurun_out/ncu_pair.log 2>&1; tail -1 gpurun_out/ncu_pair.log
