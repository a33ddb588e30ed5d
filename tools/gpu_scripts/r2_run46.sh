#!/bin/bash
# round 2, call 46: ncu --set full (source) of k_sfx (c5) and of the current k_ctile2 (c3-client slice)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx --launch-skip 1 -c 1 -o gpurun_out/r02_sfx_c5_v2 python tools/prof_search.py c5 > gpurun_out/r2at_ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ctile2 --launch-skip 1 -c 1 -o gpurun_out/r02_ctile2_v3 python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2at_ncu2.log 2>&1
echo done
