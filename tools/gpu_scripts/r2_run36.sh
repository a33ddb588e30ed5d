#!/bin/bash
# round 2, call 36: tile loop T by FMNMX3 (T3, default build) vs per-pair T2 (ab/lib_T2.so); ncu of T3 k_tile and the RT4N kernel
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in T2 T3 T2 T3 T2 T3; do echo "variant=$v" >> gpurun_out/r2aj.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,c1_set,pareto --reps 1 >> gpurun_out/r2aj.jsonl 2>&1; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4_v3 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2aj_ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_rt4n python tools/prof_search.py c4 --shard 5 64 --weights 1,1:2,1:1,2 > gpurun_out/r2aj_ncu2.log 2>&1
echo done
