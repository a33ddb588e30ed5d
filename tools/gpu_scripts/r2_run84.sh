#!/bin/bash
# round 2, call 84: final build -- full GPU suite, smoke, bench, launch list, ncu of the bench kernel, whole-space checks
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2cf_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2cf_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2cf_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2cf_bench.json 2> gpurun_out/r2cf_bench.err
timeout 900 python tools/full_check.py c3 c5 c4 > gpurun_out/r2cf_full.jsonl 2> gpurun_out/r2cf_full.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2cf_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/r2cf_ncu2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4_v7 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2cf_ncu1.log 2>&1
timeout 300 python tools/time_slices.py c4 --sets c1_set,c5_sweep,w11_21_12,eight,pareto,w11 --reps 1 > gpurun_out/r2cf_sets.jsonl 2>&1
echo done
