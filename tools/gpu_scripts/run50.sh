# ncu of the subset-DP phase-1 kernel on the literal per-client c4; c5 DP timing
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python tools/dp_c4client.py c5 gpu | cut -c1-300
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pf_items -c 1 \
   -o gpurun_out/prof_pf_items_c4client python tools/dp_c4client.py 2>&1 | tail -1 | cut -c1-200
ncu -i gpurun_out/prof_pf_items_c4client.ncu-rep --page source --csv --print-source sass > gpurun_out/pf_items_sass.csv 2>/dev/null
