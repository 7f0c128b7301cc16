#!/bin/bash
# A/B of two library builds: parity probe + C2 launch lists
timeout 300 python tools/dbg_fit.py > gpurun_out/it_dbg.log 2>&1; tail -3 gpurun_out/it_dbg.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/it_launches.csv python tools/fit_c2.py 2 > /dev/null 2>&1
DT_LIB_PATH=$PWD/paper_conf_ipps_metzgd23_b200/libdt_m2.so timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/it_launches_m2.csv python tools/fit_c2.py 2 > /dev/null 2>&1
