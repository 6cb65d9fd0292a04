#!/bin/bash
# A/B prebuilt libraries on the general-path lines of bench_modes.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for n in ${NAMES:-base new}; do
  cp scripts/abl/lib_$n.so paper_conf_ipps_boyermk13_b200/libgrophecy.so
  python scripts/bench_modes.py 2>&1 | grep -E "best_general|c3s|c3h" | sed "s/^/$n /" | cut -c1-100
done
