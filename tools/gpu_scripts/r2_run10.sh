#!/bin/bash
# round 2, call 10: warp-uniform rare paths in the tile loop; n = 16 per-client certificate on the device DP
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python tools/time_slices.py c4 --sets c4,w11,c1_set,c5_sweep,w10,pareto --reps 2 > gpurun_out/r2j_slices.jsonl 2>&1
timeout 600 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 >> gpurun_out/r2j_slices.jsonl 2>&1
timeout 1200 python -m pytest tests/test_gpu_dp.py tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_edge.py -q > gpurun_out/r2j_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2j_tests.log
echo done
