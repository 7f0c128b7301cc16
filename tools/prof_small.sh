#!/bin/bash
# ncu full captures of the per-level small kernels at a deep C2 level (development aid)
for k in fused_general_kernel chunk_plan_kernel goleft_kernel select_kernel number_kernel; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:$k -s ${SKIP:-10} -c 1 \
    -o gpurun_out/ps_$k python tools/fit_c2.py 1 > /dev/null 2>&1
done
ls -la gpurun_out/ps_*
