#!/bin/bash
# round 2, call 45: E as (E_p + A_e) + (B_e + C_e) (BCE) at 512 / 384 threads, and 384 threads alone, vs current (B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B B512 B384 T384 B B512 B384 T384; do echo "variant=$v" >> gpurun_out/r2as.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,pareto --reps 1 >> gpurun_out/r2as.jsonl 2>&1; done
echo done
