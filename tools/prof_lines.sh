mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function \
  -k regex:'^(scan_single_kernel|partition_kernel|part_agg_kernel|rs_scatter_kernel)$' --launch-skip 0 --launch-count 8 -o /tmp/lines -f \
  python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse --c3-rows 0 > gpurun_out/lines_ncu.log 2>&1
for k in scan_single_kernel partition_kernel part_agg_kernel rs_scatter_kernel; do
  python tools/ncu_lines.py /tmp/lines.ncu-rep "$k" 45 > gpurun_out/lines_$k.txt 2>&1
done
