# suffix kernel: parity, then c5 timings (sfx vs pair)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_sfx.py -x -q 2>&1 | tail -15
SCHED_KERNEL=sfx timeout 300 python tools/time_search.py c5 0 68719476736 --reps 2
SCHED_KERNEL=dfs timeout 300 python tools/time_search.py c5 0 8589934592 --reps 1
SCHED_KERNEL=sfx timeout 600 python tools/time_search.py c5 --reps 2
