# full gpu suite + ncu of the suffix kernel on a feasible-dense c5 window
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
SCHED_KERNEL=sfx timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sfx -c 1 \
   -o gpurun_out/prof_sfx_v1_c5 python tools/prof_search.py c5 200000000000 17179869184 2>&1 | tail -3
