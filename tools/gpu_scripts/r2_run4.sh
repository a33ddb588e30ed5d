#!/bin/bash
# round 2, call 4: ctile2 capacity failure debug; RT vs compiled weight timing; full GPU suite (no -x)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python tools/debug_case.py > gpurun_out/r2d_debug.log 2>&1
timeout 600 python tools/time_slices.py c4 --sets w11,w10,w10_01,w11_21_12 --reps 1 > gpurun_out/r2d_slices.jsonl 2>&1
SCHED_TILE_RT=1 timeout 600 python tools/time_slices.py c4 --sets c4,w11,w10 --reps 1 >> gpurun_out/r2d_slices.jsonl 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2d_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2d_gputests.log
echo done
