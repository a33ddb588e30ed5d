#!/bin/bash
# round 2, call 25: how much of the c4 slice is the partition walk (tiles skipped: SCHED_B0=10)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for m in 2 10 2 10; do echo "b0mode=$m" >> gpurun_out/r2y.jsonl; SCHED_SO_PATH=ab/lib_X.so SCHED_B0=$m timeout 300 python tools/time_slices.py c4 --sets c4 --reps 1 >> gpurun_out/r2y.jsonl 2>&1; done
echo done
