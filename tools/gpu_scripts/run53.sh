# subset-DP phase 1 with fp64 shared-memory tables: register budget variants
for v in ""; do
  rm -f paper_conf_sc_weaverkmeh0m24_b200/build_obj/dp_front* paper_conf_sc_weaverkmeh0m24_b200/libsched.so
  SCHED_NVCC_EXTRA="$v" python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
  echo "variant [$v]"
  python tools/dp_c4client.py | cut -c1-120
done
timeout 900 python -m pytest tests/test_gpu_dp.py -q -k "not 14" 2>&1 | tail -2
