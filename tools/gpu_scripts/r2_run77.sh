#!/bin/bash
# round 2, call 77: T1 = max3(lp.x, T_l, A_t) (X3) vs T_p then max (B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B X3 B X3 B X3; do echo "variant=$v" >> gpurun_out/r2by.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11 --reps 1 >> gpurun_out/r2by.jsonl 2>&1; done
echo done
