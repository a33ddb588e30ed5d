# final ncu --set full capture of the bench kernel (current build) + launch list of the bench command
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tile -s 1 -c 1 \
   -o gpurun_out/prof_tile_v7_c4 python tools/prof_search.py c4 100000000000000 549755813888 2>&1 | tail -1 | cut -c1-100
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01_v5.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; ls -la gpurun_out/launches_r01_v5.csv
