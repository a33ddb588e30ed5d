#!/bin/bash
# round 2, call 21: ncu --set full of k_ctile2 (c3-client 1/64 slice) and k_tile (c4 slice), current build
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ctile2 --launch-skip 1 -c 1 -o gpurun_out/r02_ctile2_v2 python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2u_ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile --launch-skip 1 -c 1 -o gpurun_out/r02_tile_c4_v2 python tools/prof_search.py c4 --shard 5 64 > gpurun_out/r2u_ncu2.log 2>&1
echo done
