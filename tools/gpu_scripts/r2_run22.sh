#!/bin/bash
# round 2, call 22: suffix kernel skips infeasible parents (E) vs D; sfx parity
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in D E D E; do echo "variant=$v" >> gpurun_out/r2v.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2v.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_E.so timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py -q -k "sfx or c5" > gpurun_out/r2v_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2v_tests.log
echo done
