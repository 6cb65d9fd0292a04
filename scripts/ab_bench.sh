#!/bin/bash
# A/B prebuilt libraries (scripts/abl/lib_<name>.so) on the full bench
# (10^9 candidates, one launch), alternating: NAMES="base new" bash scripts/ab_bench.sh
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for round in 1 2; do
  for n in ${NAMES:-base new}; do
    cp scripts/abl/lib_$n.so paper_conf_ipps_boyermk13_b200/libgrophecy.so
    echo "$n $(python bench.py --no-e2e --no-cpu-baseline --steps 10 2>&1 | tail -1 | cut -c1-120)"
  done
done
