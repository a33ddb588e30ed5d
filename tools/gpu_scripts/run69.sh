python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx -c 1 \
   -o gpurun_out/prof_sfx_v3_c5 python tools/prof_search.py c5 100000000000 60000000000 2>&1 | tail -1 | cut -c1-200
ncu -i gpurun_out/prof_sfx_v3_c5.ncu-rep --page source --csv --print-source sass > gpurun_out/sfx_v3_sass.csv 2>/dev/null; ls -la gpurun_out/sfx_v3_sass.csv
