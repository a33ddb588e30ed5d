#!/bin/bash
# round 2, call 55: k_ctile2 seed-pass size sweep on the c3-client slice (SCHED_C2_SEED="unit_log2,units_per_sm")
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for sd in "16,32" "12,32" "12,128" "14,32" "10,128" "16,8" "16,32"; do echo "seed=$sd" >> gpurun_out/r2bc.jsonl; SCHED_C2_SEED=$sd timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 2 >> gpurun_out/r2bc.jsonl 2>&1; done
echo done
