#!/bin/bash
# round 2, call 47: suffix kernel fast pass by grandparent pair tiles (PR = default build) vs parent-by-parent (PA)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2au_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2au_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -q -x -k "c5 or sfx or window or variant" > gpurun_out/r2au_tests2.log 2>&1
echo "rc=$?" >> gpurun_out/r2au_tests2.log
for v in PA PR PA PR; do echo "variant=$v" >> gpurun_out/r2au.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2au.jsonl 2>&1; done
echo done
