# line-level profile of the boundary-chunk scan at a deep level (measurement helper)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base function \
  -k regex:'^scan_kernel$' --launch-skip 10 --launch-count 1 -o /tmp/sk -f \
  python bench.py --steps 1 --warmup 0 --no-cpu --no-extra --e2e-steps 0 --no-dse --c3-rows 0 > gpurun_out/sk_ncu.log 2>&1
python tools/ncu_lines.py /tmp/sk.ncu-rep scan_kernel 40 > gpurun_out/sk_lines.txt 2>&1
ncu -i /tmp/sk.ncu-rep --page raw --csv > gpurun_out/sk_raw.csv 2>/dev/null
