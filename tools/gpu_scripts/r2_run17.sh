#!/bin/bash
# round 2, call 17: ctile2 seed pass with partition-sized sample units; fuzz parity sweep
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 > gpurun_out/r2q.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_fuzz.py tests/test_gpu_ctile2.py -q > gpurun_out/r2q_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2q_tests.log
echo done
