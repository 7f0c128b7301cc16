#!/bin/bash
# Quick GPU check after a kernel change: fit parity subset + a short fit-only bench.
TAG=${1:-q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "${2:-fit}" > gpurun_out/${TAG}_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_pytest.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu --no-extra --no-dse --c3-rows 0 --e2e-steps 2 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
if [ "${3:-0}" = 1 ]; then
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse --c3-rows 0 > gpurun_out/${TAG}_ncu_launch.log 2>&1
fi
