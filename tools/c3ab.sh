#!/bin/bash
# C3 (100M x 32, depth 16) fit time for each library given (measurement helper).
for lib in "$@"; do
  DT_LIB_PATH=$PWD/$lib timeout 900 python bench.py --no-cpu --no-dse --no-extra --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/c3ab.json 2>gpurun_out/c3ab.err
  python - "$lib" <<'PY'
import json, sys
try:
    d = json.loads(open("gpurun_out/c3ab.json").read().strip().splitlines()[-1])
    print(sys.argv[1], "C2 ms", round(d["ms_per_step"], 3), "C3 ms", round(d["c3_fit"]["ms_per_fit"], 1))
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
