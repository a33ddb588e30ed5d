# source-level ncu capture of the current tile kernel (c4 window) for the per-line instruction breakdown
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 \
   -o gpurun_out/prof_tile_v6_c4 python tools/prof_search.py c4 100000000000000 549755813888 2>&1 | tail -2
ncu -i gpurun_out/prof_tile_v6_c4.ncu-rep --page source --csv --print-source sass > gpurun_out/tile_v6_sass.csv 2>/dev/null; ls -la gpurun_out/
