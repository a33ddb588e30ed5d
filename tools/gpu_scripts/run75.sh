python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for w in c5; do timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'][:60], d['value'], d['ms_per_step'])"; done
for c in c3 c5; do python tools/time_search.py $c --reps 2 | tail -1 | cut -c1-200; done
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -2
