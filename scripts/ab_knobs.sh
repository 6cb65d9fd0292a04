#!/bin/bash
# One gpurun call: A/B of compile-time variants of the library, benched
# alternately on C4 (N = 1).  VARIANTS="- NAME=VAL,NAME=VAL ..." ("-" = defaults);
# TESTS=1 runs the GPU tests on the default build first.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
i=0
for v in ${VARIANTS:--}; do
  envs=""; [ "$v" != "-" ] && envs=$(echo "$v" | tr ',' ' ')
  env $envs python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build_v.log 2>&1 || { echo "build $v failed"; tail -5 gpurun_out/build_v.log; }
  cp paper_conf_ipps_boyermk13_b200/libgrophecy.so /tmp/lib_v$i.so
  i=$((i+1))
done
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1
if [ -n "$TESTS" ]; then timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log; fi
for rep in 1 2 ${EXTRA_REPS}; do
  i=0
  for v in ${VARIANTS:--}; do
    echo "$v: $(GROPHECY_LIB=/tmp/lib_v$i.so timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]/1e9,1), d["best"]["index"])')"
    i=$((i+1))
  done
done
if [ -n "$SEG" ]; then
  i=0
  for v in ${VARIANTS:--}; do
    echo "== seg $v"; GROPHECY_LIB=/tmp/lib_v$i.so timeout 300 python scripts/segbench.py c4 3 | python -c '
import json,sys
print(" ".join(str(round(json.loads(l)["cand_per_s"]/1e9)) for l in sys.stdin))'
    i=$((i+1))
  done
fi
