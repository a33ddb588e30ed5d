# super-tile pre-filter: parity + bench
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_r42.json 2> gpurun_out/bench_r42.err; tail -1 gpurun_out/bench_r42.json | cut -c1-400
python - <<'PY' 2>&1 | tail -2
import json; d=json.loads(open("gpurun_out/bench_r42.json").read().strip().splitlines()[-1]); print(d["value"], d["roofline"]["frac"], d["n_refined_timed"] if "n_refined_timed" in d else d["config"].get("n_refined_timed"))
PY
