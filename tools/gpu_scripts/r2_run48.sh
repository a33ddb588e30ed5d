#!/bin/bash
# round 2, call 48: ncu --set full (source) of the suffix kernel with grandparent pair tiles (c5)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx --launch-skip 1 -c 1 -o gpurun_out/r02_sfx_c5_v3 python tools/prof_search.py c5 > gpurun_out/r2av_ncu1.log 2>&1
echo done
