#!/bin/bash
# round 2, call 27: tile kernel 512 / 640 / 768 threads x 1 CTA per SM
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in T512 T640 T768 T512 T640 T768; do echo "variant=$v" >> gpurun_out/r2aa.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,c1_set --reps 1 >> gpurun_out/r2aa.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_T512.so timeout 1200 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_scores32.py -q > gpurun_out/r2aa_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2aa_tests.log
echo done
