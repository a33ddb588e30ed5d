python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
SCHED_KERNEL=generic python tools/time_search.py c2 --reps 3 | tail -1 | cut -c1-160
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -2
