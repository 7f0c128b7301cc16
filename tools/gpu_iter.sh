#!/bin/bash
# development iteration on the GPU box: parity probe, launch list, ncu of the fused pass
set -x
timeout 300 python tools/dbg_fit.py > gpurun_out/it_dbg.log 2>&1
tail -4 gpurun_out/it_dbg.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/it_launches.csv python tools/fit_c2.py 2 > /dev/null 2>&1
if [ "$1" == "full" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fused_kernel|level_agg" -s 12 -c 2 -o gpurun_out/it_prof python tools/fit_c2.py 2 > gpurun_out/it_ncu.log 2>&1
fi
