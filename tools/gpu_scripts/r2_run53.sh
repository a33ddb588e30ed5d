#!/bin/bash
# round 2, call 53: staircase screen before the weight screen for compiled sets (SF) vs current (B); ncu of k_sfx<7> (c5)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in B SF B SF B SF; do echo "variant=$v" >> gpurun_out/r2ba.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11 --reps 1 >> gpurun_out/r2ba.jsonl 2>&1; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx --launch-skip 1 -c 1 -o gpurun_out/r02_sfx_c5_v4 python tools/prof_search.py c5 > gpurun_out/r2ba_ncu.log 2>&1
echo done
