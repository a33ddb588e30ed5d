#!/bin/bash
# round 2, call 71: guided units in the tile kernel (SCHED_TILE_GUIDE g: the last 1/8 of the range in 2^g-times smaller units)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for g in 0 3 2 4 0 3; do for sl in 64 512; do echo "guide=$g slices=$sl" >> gpurun_out/r2bs.jsonl; SCHED_TILE_GUIDE=$g timeout 300 python tools/time_slices.py c4 --sets c4 --reps 2 --slices $sl >> gpurun_out/r2bs.jsonl 2>&1; done; done
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_overflow.py tests/test_gpu_nccl.py -q -x > gpurun_out/r2bs_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bs_tests.log
echo done
