#!/bin/bash
# A/B two prebuilt libgrophecy.so files (scripts/abl/lib_<name>.so) on the
# C4 segment benchmark, alternating: usage NAMES="base new" bash scripts/ab_libs.sh
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for round in 1 2; do
  for n in ${NAMES:-base new}; do
    cp scripts/abl/lib_$n.so paper_conf_ipps_boyermk13_b200/libgrophecy.so
    echo "$n $(python scripts/segbench.py c4 5 | tail -1)"
  done
done
