#!/bin/bash
# round 2, call 3: group-table PER_CLIENT tile kernel (path 6) parity + timing; (1,0) tie-flood fix timing
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ctile2.py -q -x > gpurun_out/r2c_ctile2.log 2>&1
echo "rc=$?" >> gpurun_out/r2c_ctile2.log
timeout 300 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,w11 --reps 2 > gpurun_out/r2c_slices.jsonl 2>&1
timeout 600 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 > gpurun_out/r2c_c3client.jsonl 2>&1
SCHED_KERNEL=ctile timeout 600 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 1 --slices 1024 >> gpurun_out/r2c_c3client.jsonl 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2c_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2c_gputests.log
echo done
