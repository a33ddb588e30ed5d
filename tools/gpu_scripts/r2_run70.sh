#!/bin/bash
# round 2, call 70: tile-kernel units per warp (SCHED_TILE_UPW) at 1/64 (R = 1) and 1/512 (a rank's share at R = 8)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for u in 16 32 64 128 16; do for sl in 64 512; do echo "upw=$u slices=$sl" >> gpurun_out/r2br.jsonl; SCHED_TILE_UPW=$u timeout 300 python tools/time_slices.py c4 --sets c4 --reps 2 --slices $sl >> gpurun_out/r2br.jsonl 2>&1; done; done
echo done
