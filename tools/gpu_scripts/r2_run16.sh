#!/bin/bash
# round 2, call 16: seed-pass cost on the per-client and tile kernels
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for u in 128 32 8; do echo "seed_units_per_sm=$u" >> gpurun_out/r2p.jsonl; SCHED_SEED_UNITS_PER_SM=$u timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 >> gpurun_out/r2p.jsonl 2>&1; done
for u in 128 32; do echo "seed_units_per_sm=$u" >> gpurun_out/r2p.jsonl; SCHED_SEED_UNITS_PER_SM=$u timeout 300 python tools/time_slices.py c4 --sets c4 --reps 2 >> gpurun_out/r2p.jsonl 2>&1; done
timeout 600 nsys --version > /dev/null 2>&1 || echo "no nsys" >> gpurun_out/r2p.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2p_launches_c3client.csv 2>&1
echo done
