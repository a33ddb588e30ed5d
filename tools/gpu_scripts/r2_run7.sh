#!/bin/bash
# round 2, call 7: global b0 F filter; parity; timings; ncu captures (tile c4 slice, ctile2 c3-client slice, bench launch list)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_edge.py tests/test_gpu_ctile2.py tests/test_gpu_variants.py -q > gpurun_out/r2g_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2g_tests.log
timeout 900 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,w10,w11 --reps 1 > gpurun_out/r2g_slices.jsonl 2>&1
for m in LAZY EAGER; do CUDA_MODULE_LOADING=$m timeout 300 python tools/dp_cold.py c4 >> gpurun_out/r2g_dp_cold.jsonl 2>&1; done
CUDA_MODULE_LOADING=LAZY timeout 300 python tools/dp_cold.py c4 --after-search >> gpurun_out/r2g_dp_cold.jsonl 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2g_ncu_tile.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ctile2 --launch-skip 1 -c 1 -o gpurun_out/r02_ctile2_c3client python tools/prof_search.py c3 --scope 0 --shard 5 1024 > gpurun_out/r2g_ncu_ctile2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r2g_ncu_launches.log 2>&1
echo done
