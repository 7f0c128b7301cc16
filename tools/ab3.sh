#!/bin/bash
# Bench-only A/B of libdt variants with the presort time (measurement helper).
# usage: bash tools/ab3.sh <tag> lib1 lib2 ...
TAG=$1; shift
mkdir -p gpurun_out
for rep in 1 2; do
for lib in "$@"; do
  DT_LIB_PATH=$lib timeout 600 python bench.py --no-cpu --no-dse --no-extra --c3-rows 0 --steps 30 --e2e-steps 1 > gpurun_out/${TAG}_b.json 2> gpurun_out/${TAG}_b.err
  python - "$lib" gpurun_out/${TAG}_b.json <<'PY' | tee -a gpurun_out/${TAG}_ab.txt
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    bk = d["roofline"]["by_kernel"]
    print(sys.argv[1], round(d["value"] / 1e9, 2), "G/s", round(d["ms_per_step"], 3), "ms", "presort", bk["presort_sort"]["ms_per_step"], "fused", bk["fused"]["ms_per_step"])
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
done
