#!/bin/bash
# round 2, call 8: DevParams in global memory for slow paths (no stack copy); b0 mode matrix; parity
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 600 python tools/time_slices.py c4 --sets c4,w11,c1_set --reps 2 > gpurun_out/r2h_slices.jsonl 2>&1
for m in 0 1 2 3; do echo "b0mode=$m" >> gpurun_out/r2h_slices.jsonl; SCHED_B0=$m timeout 300 python tools/time_slices.py c4 --sets w10 --reps 1 >> gpurun_out/r2h_slices.jsonl 2>&1; done
timeout 1200 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_edge.py -q > gpurun_out/r2h_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2h_tests.log
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none -k regex:k_tile --launch-skip 1 -c 1 --csv python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2h_ncu_tile.csv 2>&1
echo done
