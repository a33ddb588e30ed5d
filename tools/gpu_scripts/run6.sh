timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
ncu --set full --clock-control none --import-source on -k regex:k_tile -c 1 -o gpurun_out/prof_tile_v2_c4 python tools/prof_search.py c4 30000000000000 68719476736 > gpurun_out/ncu_tile_v2.log 2>&1; tail -2 gpurun_out/ncu_tile_v2.log
