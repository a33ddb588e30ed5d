#!/bin/bash
# round 2, call 23: ctile2 seed-pass shapes
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for sd in "10,128" "14,64" "16,32" "16,64" "18,16" "20,4"; do echo "seed=$sd" >> gpurun_out/r2w.jsonl; SCHED_SO_PATH=ab/lib_F.so SCHED_C2_SEED=$sd timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 >> gpurun_out/r2w.jsonl 2>&1; done
echo done
