#!/bin/bash
# round 2, call 43 (measurement only): cost of the per-partition setup of k_tile -- the same partition scored
# again without the successor (NS1) and without the group-record loads (NS2), vs the product (B); results of NS* are wrong
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B NS1 NS2 B NS1 NS2; do echo "variant=$v" >> gpurun_out/r2aq.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4 --reps 1 >> gpurun_out/r2aq.jsonl 2>&1; done
echo done
