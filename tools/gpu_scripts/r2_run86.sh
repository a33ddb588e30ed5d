#!/bin/bash
# round 2, call 86: tile seed-pass size (units per SM) at 1/512 (a rank's share at R = 8) and 1/64
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for u in 128 64 32 16 128; do for sl in 512 64; do echo "seed_upsm=$u slices=$sl" >> gpurun_out/r2cg.jsonl; SCHED_SEED_UNITS_PER_SM=$u timeout 300 python tools/time_slices.py c4 --sets c4 --reps 2 --slices $sl >> gpurun_out/r2cg.jsonl 2>&1; done; done
echo done
