# ncu of the suffix kernel on the full c5 search (skip the seed pass launch)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
SCHED_KERNEL=sfx timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx -s 1 -c 1 \
   -o gpurun_out/prof_sfx_v2_c5full python tools/prof_search.py c5 2>&1 | tail -3
