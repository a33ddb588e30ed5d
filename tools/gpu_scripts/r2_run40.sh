#!/bin/bash
# round 2, call 40: bench of the committed build + ncu of the bench kernel (source level) + launch list
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2an_bench.json 2> gpurun_out/r2an_bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4_v4 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2an_ncu1.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2an_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/r2an_ncu2.log 2>&1
echo done
