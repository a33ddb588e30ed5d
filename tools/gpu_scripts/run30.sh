# full-size timings of every BASELINE workload + ncu launch list of the bench step
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for c in c1 c2 c3 c5; do python tools/time_search.py $c --reps 2 | tail -1 | cut -c1-420; done
SCHED_KERNEL=generic python tools/time_search.py c2 --reps 1 | cut -c1-300
timeout 900 python bench.py --full 2>&1 | tail -1 | cut -c1-800
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01_v3.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1; tail -1 gpurun_out/ncu_bench.log | cut -c1-200
