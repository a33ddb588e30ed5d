#!/bin/bash
# round 2, call 78: final build -- full GPU suite, smoke, bench, launch list, ncu of the bench kernel, whole-space checks
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2bz_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bz_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bz_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2bz_bench.json 2> gpurun_out/r2bz_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bz_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/r2bz_ncu2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4_v6 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2bz_ncu1.log 2>&1
timeout 900 python tools/full_check.py c3 c5 c4 > gpurun_out/r2bz_full.jsonl 2> gpurun_out/r2bz_full.err
echo done
