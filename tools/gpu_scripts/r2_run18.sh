#!/bin/bash
# round 2, call 18: lazy fp64 in the per-client slow paths; fuzz sweep; c3-client timing
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 > gpurun_out/r2r.jsonl 2>&1
SCHED_KERNEL=ctile timeout 300 python tools/time_slices.py c2 --sets c4 --reps 2 >> gpurun_out/r2r.jsonl 2>&1
timeout 300 python tools/time_search.py c2 --reps 2 >> gpurun_out/r2r.jsonl 2>&1
timeout 1800 python -m pytest tests/test_gpu_fuzz.py tests/test_gpu_ctile2.py tests/test_gpu_edge.py -q > gpurun_out/r2r_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2r_tests.log
echo done
