#!/bin/bash
# round 2, call 66: whole-space exhaustive searches (c3, c5, c4 in 64 slices) vs the committed exact certificates
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python tools/full_check.py c3 c5 c4 > gpurun_out/r2bn_full.jsonl 2> gpurun_out/r2bn_full.err
echo done
