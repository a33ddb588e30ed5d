#!/bin/bash
# round 2, call 35: run-time weight kernels without b = 0 weights (WS_RTN / WS_RT4N); NCCL one-rank tests
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python tools/time_slices.py c4 --sets c4,w11_21_12,eight --reps 2 > gpurun_out/r2ai.jsonl 2>&1
SCHED_TILE_RT=1 timeout 600 python tools/time_slices.py c4 --sets c4,w11 --reps 2 >> gpurun_out/r2ai.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_nccl.py tests/test_gpu_tile_weights.py tests/test_gpu_fuzz.py -q > gpurun_out/r2ai_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ai_tests.log
echo done
