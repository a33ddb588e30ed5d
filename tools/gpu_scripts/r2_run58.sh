#!/bin/bash
# round 2, call 58: overflowing passes stop early; pass 2 re-bucketed to the overflowing pass's span (seeded too):
# forced-overflow tests, the tiny-seed pathology (SCHED_C2_SEED=16,8: 163 s before), regression timing, parity
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_overflow.py -q -x -rs > gpurun_out/r2bf_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bf_tests.log
SCHED_C2_SEED=16,8 timeout 400 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 1 > gpurun_out/r2bf.jsonl 2>&1
timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 2 >> gpurun_out/r2bf.jsonl 2>&1
timeout 300 python tools/time_slices.py c4 --sets c4 --reps 2 >> gpurun_out/r2bf.jsonl 2>&1
timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2bf.jsonl 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py tests/test_gpu_ctile2.py tests/test_gpu_sfx.py -q -x > gpurun_out/r2bf_tests2.log 2>&1
echo "rc=$?" >> gpurun_out/r2bf_tests2.log
echo done
