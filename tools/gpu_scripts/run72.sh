python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python tools/dp_c4client.py c5 gpu | cut -c1-100
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dp_c5.csv python tools/dp_c4client.py c5 gpu > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/launches_dp_c5.csv gpurun_out/launches_dp_c5.md; head -12 gpurun_out/launches_dp_c5.md
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_dp_level -s 12 -c 1 -o gpurun_out/prof_dp_level_c5 python tools/dp_c4client.py c5 gpu > /dev/null 2>&1; ls gpurun_out/prof_dp_level_c5.ncu-rep
