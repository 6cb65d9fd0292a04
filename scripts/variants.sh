#!/bin/bash
# Build + segbench several compile-time variants in one gpurun call.
# usage: VARIANTS="A:GROPHECY_VAL=512,GROPHECY_MINB=2 B:..." bash scripts/variants.sh [config]
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
cfg=${1:-c4}
for v in $VARIANTS; do
  name=${v%%:*}; envs=${v#*:}
  env $(echo $envs | tr ',' ' ') python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build_$name.log 2>&1 || { echo "$name build failed"; continue; }
  python scripts/segbench.py $cfg 5 > gpurun_out/seg_$name.txt 2>&1
  echo "$name $(tail -1 gpurun_out/seg_$name.txt)"
done
