#!/bin/bash
# round 2, call 57: k_ctile2 seed pass by whole partitions (units of 2^24 / 2^22 / 2^20 ...) instead of 2^16 pieces
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for sd in "16,32" "24,1" "24,2" "22,2" "22,8" "20,8" "18,16"; do echo "seed=$sd" >> gpurun_out/r2be.jsonl; SCHED_C2_SEED=$sd timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 2 >> gpurun_out/r2be.jsonl 2>&1; done
echo done
