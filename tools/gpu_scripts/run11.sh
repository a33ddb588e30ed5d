cat > case_tmp.py <<'PY'
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import make_profile, Query
prof = make_profile(7, levels=(25, 50, 75, 100), seed=3)
q = Query(7, 7, 7, (25, 50, 75, 100), 1, (), True)
r = S.Scheduler(prof).search(q)
print(r.stats, r.pareto_indices)
PY
timeout 600 compute-sanitizer --tool memcheck --show-backtrace device python case_tmp.py 2>&1 | head -60
