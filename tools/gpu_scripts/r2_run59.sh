#!/bin/bash
# round 2, call 59: ctile2 seed by whole tiles (SCHED_C2_SEED_TILES=1, default) vs index pieces (=0); unseeded c3-client;
# overflow tests (revised); tiny-seed pathology
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in 0 1 0 1; do echo "seed_tiles=$v" >> gpurun_out/r2bg.jsonl; SCHED_C2_SEED_TILES=$v timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 1 >> gpurun_out/r2bg.jsonl 2>&1; done
echo "noseed" >> gpurun_out/r2bg.jsonl; SCHED_NO_SEED=1 timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 1 >> gpurun_out/r2bg.jsonl 2>&1
echo "noseed c4" >> gpurun_out/r2bg.jsonl; SCHED_NO_SEED=1 timeout 300 python tools/time_slices.py c4 --sets c4 --reps 1 >> gpurun_out/r2bg.jsonl 2>&1
echo "tiles seed=16,8" >> gpurun_out/r2bg.jsonl; SCHED_C2_SEED=16,8 timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 1 >> gpurun_out/r2bg.jsonl 2>&1
timeout 1200 python -m pytest tests/test_gpu_overflow.py tests/test_gpu_ctile2.py -q -rs > gpurun_out/r2bg_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bg_tests.log
echo done
