#!/bin/bash
# per-kernel ncu launch lists of the fit bench for several libdt variants (measurement
# helper, not part of the library): gpurun_out/ncu_<tag>.csv
i=0
for lib in "$@"; do
  i=$((i+1))
  DT_LIB_PATH=$lib timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum \
    --clock-control none --csv --log-file gpurun_out/ncu_v$i.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse > /dev/null 2>&1
done
