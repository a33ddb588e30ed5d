#!/bin/bash
# round 2, call 65: 256-configuration tiles with per-sub-tile corners (T256b) vs 64-configuration tiles (N256)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in N256 T256b N256 T256b; do echo "variant=$v" >> gpurun_out/r2bm.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11 --reps 1 >> gpurun_out/r2bm.jsonl 2>&1; done
echo done
