# tile kernel block shape / register budget sweep (c4 windows)
for v in "" "-DSCHED_TILE_THREADS=192 -DSCHED_TILE_MINB=2" "-DSCHED_TILE_THREADS=384 -DSCHED_TILE_MINB=1" "-DSCHED_TILE_THREADS=256 -DSCHED_TILE_MINB=1"; do
  rm -f paper_conf_sc_weaverkmeh0m24_b200/build_obj/tile_* paper_conf_sc_weaverkmeh0m24_b200/libsched.so
  SCHED_NVCC_EXTRA="$v" python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
  echo "variant [$v]"
  python tools/time_search.py c4 0 3298534883328 --reps 2 | cut -c1-200
  python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-200
done
