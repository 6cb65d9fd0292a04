#!/bin/bash
# A/B prebuilt libraries (scripts/abl/lib_<name>.so) on the best-mode lines of
# bench_modes (C4 sample, C3, C3s, C3h), two alternating rounds.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
for round in 1 2; do
  for n in ${NAMES:-base new}; do
    cp scripts/abl/lib_$n.so paper_conf_ipps_boyermk13_b200/libgrophecy.so
    python scripts/bench_modes.py 2>&1 | grep -E '"mode": "best"|best_general' | sed "s/^/$n /" | cut -c1-110
  done
done
