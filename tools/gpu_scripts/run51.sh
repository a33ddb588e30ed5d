python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dp_c4client_v2.csv python tools/dp_c4client.py > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/launches_dp_c4client_v2.csv gpurun_out/launches_dp_c4client_v2.md; cat gpurun_out/launches_dp_c4client_v2.md | head -20
