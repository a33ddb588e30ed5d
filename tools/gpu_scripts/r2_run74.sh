#!/bin/bash
# round 2, call 74: suffix fast pass with the odometer over great-grandparents (G3 = default build) vs grandparents (GP)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
SCHED_SO_PATH=ab/lib_G3.so timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_overflow.py -q -x > gpurun_out/r2bv_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bv_tests.log
for v in GP G3 GP G3; do echo "variant=$v" >> gpurun_out/r2bv.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2bv.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_G3.so timeout 300 python tools/full_check.py c5 >> gpurun_out/r2bv.jsonl 2>&1
echo done
