#!/bin/bash
# round 2, call 32: suffix kernel 256x2 vs 512x1
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in S256 S512 S256 S512; do echo "variant=$v" >> gpurun_out/r2af.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2af.jsonl 2>&1; done
echo done
