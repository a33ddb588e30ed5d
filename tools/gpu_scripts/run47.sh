# round-1 final: build, full GPU parity, smoke, bench (with subset-DP time-to-optimal), ncu launch list of the bench
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_r47.json 2> gpurun_out/bench_r47.err; tail -1 gpurun_out/bench_r47.json | cut -c1-300
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01_v4.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench_v4.log 2>&1; tail -1 gpurun_out/ncu_bench_v4.log | cut -c1-100
