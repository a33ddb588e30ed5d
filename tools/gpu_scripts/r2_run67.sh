#!/bin/bash
# round 2, call 67: T = max3(T_p, max(A,B) table, C) (AB) vs current (B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B AB B AB B AB; do echo "variant=$v" >> gpurun_out/r2bo.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11,pareto --reps 1 >> gpurun_out/r2bo.jsonl 2>&1; done
echo done
