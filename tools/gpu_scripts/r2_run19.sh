#!/bin/bash
# round 2, call 19: A/B of the per-client kernel changes (c3-client slice)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in A B C A B C; do echo "variant=$v" >> gpurun_out/r2s.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 1 >> gpurun_out/r2s.jsonl 2>&1; done
echo done
