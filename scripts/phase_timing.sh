#!/bin/bash
# One gpurun call: per-phase timing of the sweep kernel (diagnostic build) and
# the bench line, for each build variant in VARIANTS ("NAME=VAL,NAME=VAL ..."
# sets of GROPHECY_* macros; "-" = defaults).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for v in ${VARIANTS:--}; do
  envs=""; [ "$v" != "-" ] && envs=$(echo "$v" | tr ',' ' ')
  echo "### variant $v"
  env $envs GROPHECY_PHASE_TIMING=1 python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || tail gpurun_out/build.log
  for c in ${CONFIGS:-c4}; do echo "== $c"; timeout 300 python scripts/phase_timing.py $c; done
  env $envs python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1
  timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-170
  if [ -n "$TESTS" ]; then timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log; fi
done
