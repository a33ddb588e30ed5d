python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1

timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_ctile -c 1 \
   -o gpurun_out/prof_ctile_c2_v4 python tools/prof_search.py c2 2>&1 | tail -1 | cut -c1-200
ncu -i gpurun_out/prof_ctile_c2_v4.ncu-rep --page source --csv --print-source sass > gpurun_out/ctile_c2_v4_sass.csv 2>/dev/null; ls -la gpurun_out/ctile_c2_v4_sass.csv
