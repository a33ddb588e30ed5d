python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_sfx.py -x -q 2>&1 | tail -4
SCHED_KERNEL=sfx timeout 600 python tools/time_search.py c5 --reps 3 | cut -c1-400
