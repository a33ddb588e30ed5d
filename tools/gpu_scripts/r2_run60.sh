#!/bin/bash
# round 2, call 60: k_ctile2 tile-seed size sweep (units per SM) on the c3-client slice
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for sd in "16,32" "16,8" "16,16" "16,64" "16,128" "16,32"; do echo "seed=$sd" >> gpurun_out/r2bh.jsonl; SCHED_C2_SEED=$sd timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 2 >> gpurun_out/r2bh.jsonl 2>&1; done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bh_launches.csv python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2bh_ncu.log 2>&1
echo done
