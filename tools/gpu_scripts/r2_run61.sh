#!/bin/bash
# round 2, call 61: k_ctile2 seed pass refreshing thresholds / staircase every 4 steps (RF) vs HEAD (H); seeds 32 / 64 per SM
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in "H 16,32" "RF 16,32" "H 16,64" "RF 16,64" "H 16,32" "RF 16,32" "H 16,64" "RF 16,64"; do set -- $v; echo "variant=$1 seed=$2" >> gpurun_out/r2bi.jsonl; SCHED_C2_SEED=$2 SCHED_SO_PATH=ab/lib_$1.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 2 >> gpurun_out/r2bi.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_RF.so timeout 1200 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_overflow.py -q -x > gpurun_out/r2bi_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bi_tests.log
echo done
