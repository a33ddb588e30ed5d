#!/bin/bash
# round 2, call 5: re-bucketed overflow re-run; WS_C1 / WS_SWEEP tile instantiations; b0 partition skip
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python tools/debug_case.py > gpurun_out/r2e_debug.log 2>&1
timeout 900 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,w10,w10_01,eight --reps 1 > gpurun_out/r2e_slices.jsonl 2>&1
timeout 1500 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_sfx.py -q > gpurun_out/r2e_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2e_tests.log
echo done
