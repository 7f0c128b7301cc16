#!/bin/bash
# build, then run a command on the GPU box only if the build succeeded
set -e
cd "$(dirname "$0")/.."
python paper_conf_ipps_metzgd23_b200/build.py > /tmp/build.log 2>&1 || { grep -E "error" /tmp/build.log | head; echo BUILD FAILED; exit 1; }
timeout ${GPU_TIMEOUT:-2000} /usr/local/graft/bin/gpurun --timeout ${GPU_LIMIT:-1200} -- "$1" 2>&1 | tail -${TAILN:-12}
