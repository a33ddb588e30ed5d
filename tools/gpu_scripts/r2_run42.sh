#!/bin/bash
# round 2, call 42: tile loop unrolled by 2 (U2) / lane digits folded into shared-memory slots (SA) vs current (B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B U2 SA B U2 SA; do echo "variant=$v" >> gpurun_out/r2ap.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,pareto --reps 1 >> gpurun_out/r2ap.jsonl 2>&1; done
echo done
