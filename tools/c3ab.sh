for lib in paper_conf_ipps_metzgd23_b200/libdt_bc1024.so paper_conf_ipps_metzgd23_b200/libdt.so; do
  DT_LIB_PATH=$PWD/$lib timeout 900 python bench.py --no-cpu --no-dse --no-extra --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/c3ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/c3ab.json').read().strip().splitlines()[-1]); print('$lib', d['ms_per_step'], d['c3_fit']['ms_per_fit'])"
done
