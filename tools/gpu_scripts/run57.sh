python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for ls in 1 0; do for c in c2; do SCHED_LANE_STRIDED=$ls python tools/time_search.py $c --reps 3 | tail -1 | cut -c1-200; done; done
SCHED_LANE_STRIDED=0 SCHED_KERNEL=generic python tools/time_search.py c3 0 2000000000 | cut -c1-200
