set -x
python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err; tail -3 gpurun_out/bench_r01.err
cat gpurun_out/bench_r01.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1; tail -2 gpurun_out/bench_under_ncu.log
ncu --set full --clock-control none --import-source on -k regex:k_tile -c 1 -o gpurun_out/prof_tile_c4 python tools/prof_search.py c4 100000000000000 17179869184 > gpurun_out/ncu_tile.log 2>&1; tail -3 gpurun_out/ncu_tile.log
ncu --set full --clock-control none --import-source on -k regex:k_generic -c 1 -o gpurun_out/prof_generic_c2 python tools/prof_search.py c2 > gpurun_out/ncu_generic.log 2>&1; tail -3 gpurun_out/ncu_generic.log
