#!/bin/bash
# round 2, call 54: launch list of one c3-client slice search and one c5 search
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bb_launches_c3client.csv python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2bb_1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bb_launches_c5.csv python tools/prof_search.py c5 > gpurun_out/r2bb_2.log 2>&1
echo done
