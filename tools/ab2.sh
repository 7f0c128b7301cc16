#!/bin/bash
# A/B of libdt variants (measurement helper): fit parity tests of the LAST library given,
# then the fit bench for each library given (two rounds).
# usage: bash tools/ab2.sh <tag> <pytest -k expr> lib1 lib2 ...
TAG=$1; K=$2; shift 2
mkdir -p gpurun_out
LAST="${@: -1}"
DT_LIB_PATH=$LAST timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_scale.py -x -q -k "$K" > gpurun_out/${TAG}_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_pytest.log
tail -3 gpurun_out/${TAG}_pytest.log
for rep in 1 2; do
for lib in "$@"; do
  DT_LIB_PATH=$lib timeout 600 python bench.py --no-cpu --no-dse --no-extra --c3-rows 0 --steps 30 --e2e-steps 1 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1])
print('$lib', round(d['value']/1e9,2), 'G/s', round(d['ms_per_step'],3), 'ms', 'fused frac', round(d['roofline']['by_kernel']['fused']['frac'],3), 'fused ms', d['roofline']['by_kernel']['fused']['ms_per_step'])" | tee -a gpurun_out/${TAG}_ab.txt
done
done
