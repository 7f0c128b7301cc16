#!/bin/bash
# Source-level ncu capture of one kernel of a C2 fit (measurement helper, not part of the
# library): per-SASS-line instruction counts and stall samples -> gpurun_out/<tag>_src_*.csv
# usage: bash tools/ncu_source.sh <tag> <kernel regex> [skip] [count]
TAG=$1; K=$2; S=${3:-20}; C=${4:-1}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$K" -s $S -c $C \
  -o /tmp/${TAG}_src -f python tools/fit_c2.py 3 > gpurun_out/${TAG}_src.log 2>&1
echo "ncu exit $?" >> gpurun_out/${TAG}_src.log
ncu -i /tmp/${TAG}_src.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_src_sass.csv 2>>gpurun_out/${TAG}_src.log
ncu -i /tmp/${TAG}_src.ncu-rep --page source --csv --print-source cuda > gpurun_out/${TAG}_src_cuda.csv 2>>gpurun_out/${TAG}_src.log
ncu -i /tmp/${TAG}_src.ncu-rep --page raw --csv > gpurun_out/${TAG}_src_raw.csv 2>>gpurun_out/${TAG}_src.log
