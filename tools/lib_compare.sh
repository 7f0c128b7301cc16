#!/bin/bash
# compare libdt variants on the fit bench (measurement helper, not part of the library)
for lib in "$@"; do
  DT_LIB_PATH=$lib timeout 600 python bench.py --no-cpu --no-dse --steps 20 --e2e-steps 1 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); k=None
print('$lib', round(d['value']/1e9,2), 'G/s', round(d['ms_per_step'],3), 'ms')"
done
