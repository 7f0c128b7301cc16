mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/dse_launch.csv python tools/dse_time.py x > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:predict_dse_spec -s 1 -c 1 -o /tmp/dsefull -f python tools/dse_time.py x > /dev/null 2>&1
ncu -i /tmp/dsefull.ncu-rep --page raw --csv > gpurun_out/dse_full_raw.csv
ncu -i /tmp/dsefull.ncu-rep --page details --csv > gpurun_out/dse_full_details.csv
