#!/bin/bash
# round 2, call 63: k_ctile2 without per-tile range checks for whole-partition units (IN) vs HEAD (H)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in H IN H IN H IN; do echo "variant=$v" >> gpurun_out/r2bk.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 1 >> gpurun_out/r2bk.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_IN.so timeout 1200 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_fuzz.py tests/test_gpu_edge.py -q -x > gpurun_out/r2bk_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bk_tests.log
echo done
