#!/bin/bash
# round 2, call 39: vote-guarded tile loop (b = 0 sets) restructured like the plain loop (V = default) vs N1
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in N1 V N1 V; do echo "variant=$v" >> gpurun_out/r2am.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,w10,eight --reps 1 >> gpurun_out/r2am.jsonl 2>&1; done
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_scores32.py tests/test_gpu_variants.py -q -x > gpurun_out/r2am_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2am_tests.log
echo done
