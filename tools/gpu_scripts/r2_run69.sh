#!/bin/bash
# round 2, call 69: launch list of one rank's share of a bench step at R = 8 (shard 5 of 512), seeded and unseeded
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bq_launches_r8.csv python tools/prof_search.py c4 --shard 5 512 > gpurun_out/r2bq_1.log 2>&1
for s in 0 1 0 1; do echo "noseed=$s" >> gpurun_out/r2bq.jsonl; SCHED_NO_SEED=$s timeout 300 python tools/time_slices.py c4 --sets c4 --reps 3 --slices 512 >> gpurun_out/r2bq.jsonl 2>&1; done
echo done
