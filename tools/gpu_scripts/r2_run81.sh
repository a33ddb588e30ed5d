#!/bin/bash
# round 2, call 81: partition-wide staircase bound in the vote-guarded tile loop (sets with b = 0 weights) (VP) vs H
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in H VP H VP H VP; do echo "variant=$v" >> gpurun_out/r2cc.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c1_set,c5_sweep,eight --reps 1 >> gpurun_out/r2cc.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_VP.so timeout 1500 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_edge.py -q -x > gpurun_out/r2cc_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2cc_tests.log
echo done
