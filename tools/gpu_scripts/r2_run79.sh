#!/bin/bash
# round 2, call 79: k_ctile2 with the partition-wide staircase bound (CP) vs HEAD (H)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in H CP H CP H CP; do echo "variant=$v" >> gpurun_out/r2ca.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 1 >> gpurun_out/r2ca.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_CP.so timeout 1200 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_overflow.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2ca_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ca_tests.log
echo done
