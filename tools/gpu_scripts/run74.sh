python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for w in c2 c5; do timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'][:90], d['value'], d['ms_per_step'], d['config']['time_to_optimal_schedule_subset_dp']['device_ms'])"; done
