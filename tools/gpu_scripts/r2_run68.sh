#!/bin/bash
# round 2, call 68: split balance of the bench step over 1/2/4/8 ranks on one B200 (current build)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python tools/shard_balance.py > gpurun_out/r02_shard_balance.md 2> gpurun_out/r2bp.err
echo done
