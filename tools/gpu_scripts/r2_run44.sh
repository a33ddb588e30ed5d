#!/bin/bash
# round 2, call 44: warp-cooperative partition successor in k_tile (WS = default build) vs lane-0 walk (B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_variants.py -q -x > gpurun_out/r2ar_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ar_tests.log
for v in B WS B WS B WS; do echo "variant=$v" >> gpurun_out/r2ar.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,c1_set,pareto --reps 1 >> gpurun_out/r2ar.jsonl 2>&1; done
echo done
