# tile kernel with precomputed exact tile corners: block shape sweep
for v in "-DSCHED_TILE_THREADS=192 -DSCHED_TILE_MINB=2" "-DSCHED_TILE_THREADS=384 -DSCHED_TILE_MINB=1" "-DSCHED_TILE_THREADS=160 -DSCHED_TILE_MINB=3"; do
  rm -f paper_conf_sc_weaverkmeh0m24_b200/build_obj/tile_* paper_conf_sc_weaverkmeh0m24_b200/libsched.so
  SCHED_NVCC_EXTRA="$v" python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
  echo "variant [$v]"; grep -A2 "k_tileILi4ENS_8WS_11_21" paper_conf_sc_weaverkmeh0m24_b200/build.log | grep -i "spill\|registers"
  python tools/time_search.py c4 0 3298534883328 --reps 1 | cut -c1-160
  python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-160
done
