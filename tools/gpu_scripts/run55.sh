# generic kernel: shift / 32-bit level-digit decode; c1/c2 timing + parity
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for c in c1 c2; do python tools/time_search.py $c --reps 3 | tail -1 | cut -c1-250; done

timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
SCHED_KERNEL=generic python tools/time_search.py c3 0 2000000000 | cut -c1-200
