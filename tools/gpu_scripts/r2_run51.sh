#!/bin/bash
# round 2, call 51: suffix length 7 (SCHED_SFX_M=7) at 256x2 (P2 build) and 512x1 (S512 build) vs M = 6 (P2)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in "P2 6" "P2 7" "S512 6" "S512 7" "P2 6" "P2 7" "S512 6" "S512 7"; do set -- $v; echo "variant=$1 M=$2" >> gpurun_out/r2ay.jsonl; SCHED_SFX_M=$2 SCHED_SO_PATH=ab/lib_$1.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2ay.jsonl 2>&1; done
SCHED_SFX_M=7 SCHED_SO_PATH=ab/lib_S512.so timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py -q -x > gpurun_out/r2ay_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ay_tests.log
echo done
