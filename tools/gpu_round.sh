#!/bin/bash
# One GPU verification pass (run under gpurun from the repo root):
#   GPU tests, smoke, the default bench line, an ncu launch list of one bench step and an
#   ncu --set full capture of the fit's streaming kernels + predict.  Outputs in gpurun_out/.
# usage: gpurun --timeout 2400 -- 'bash tools/gpu_round.sh [tag] [tests=1]'
TAG=${1:-r02}
TESTS=${2:-1}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
if [ "$TESTS" = 1 ]; then
  timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/${TAG}_pytest_gpu.log 2>&1
  echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
  echo "smoke exit $?" >> gpurun_out/${TAG}_smoke.log
fi
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
echo "bench exit $?" >> gpurun_out/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse --c3-rows 0 > gpurun_out/${TAG}_ncu_launch.log 2>&1
echo "ncu launch exit $?" >> gpurun_out/${TAG}_ncu_launch.log
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
  -k regex:'fused_kernel|level_agg_kernel|rs_scatter_kernel|goleft_kernel|select_kernel' \
  --launch-count 14 -o /tmp/${TAG}_full -f \
  python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse --c3-rows 0 > gpurun_out/${TAG}_ncu_full.log 2>&1
echo "ncu full exit $?" >> gpurun_out/${TAG}_ncu_full.log
ncu -i /tmp/${TAG}_full.ncu-rep --page raw --csv > gpurun_out/${TAG}_full_raw.csv 2>/dev/null
ncu -i /tmp/${TAG}_full.ncu-rep --page details --csv > gpurun_out/${TAG}_full_details.csv 2>/dev/null
ls -la /tmp/${TAG}_full.ncu-rep >> gpurun_out/${TAG}_ncu_full.log
# predict kernels (materialised rows and the factored DSE), one launch each
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function \
  -k regex:'^(predict_col_kernel|predict_dse_spec_kernel|dse_spec_kernel|forest_predict_kernel)$' --launch-count 4 -o /tmp/${TAG}_pred -f \
  python bench.py --steps 1 --warmup 0 --no-cpu --e2e-steps 0 --dse-log2 24 --c3-rows 0 --grid-rows 0 > gpurun_out/${TAG}_ncu_pred.log 2>&1
echo "ncu pred exit $?" >> gpurun_out/${TAG}_ncu_pred.log
ncu -i /tmp/${TAG}_pred.ncu-rep --page raw --csv > gpurun_out/${TAG}_pred_raw.csv 2>/dev/null
