python tools/dp_c4client.py | cut -c1-600
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dp_c4client.csv python tools/dp_c4client.py > /dev/null 2>&1
