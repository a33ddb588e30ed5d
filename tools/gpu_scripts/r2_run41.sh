#!/bin/bash
# round 2, call 41: k_ctile2 (literal per-client c3) with T by FMNMX3, ld.shared staircase screen, staircase-first
# weight screen (C2 = default build) vs HEAD (H)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in H C2 H C2 H C2; do echo "variant=$v" >> gpurun_out/r2ao.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 1 >> gpurun_out/r2ao.jsonl 2>&1; done
timeout 1800 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_fuzz.py tests/test_gpu_edge.py -q -x > gpurun_out/r2ao_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ao_tests.log
echo done
