python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python tools/dp_prefix.py 13
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pf_items -c 1 \
   -o gpurun_out/prof_pf_items_n13_v2 python tools/dp_prefix.py 13 2>&1 | tail -1 | cut -c1-200
