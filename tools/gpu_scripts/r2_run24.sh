#!/bin/bash
# round 2, call 24: suffix kernel skips memory-infeasible subtrees (G) vs F
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in F G F G; do echo "variant=$v" >> gpurun_out/r2x.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2x.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_G.so timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_parity.py -q -k "sfx or c5 or fuzz or windows" > gpurun_out/r2x_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2x_tests.log
echo done
