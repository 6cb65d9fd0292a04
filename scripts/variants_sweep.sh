#!/bin/bash
# One gpurun call: bench several compile-time variants of the sweep kernel.
# VARIANTS="SMINB:NCH:I2F_MAGIC ..." (default "2:8:0 2:8:1")
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
for v in ${VARIANTS:-2:8:0 2:8:1}; do
  IFS=: read mb nch mg <<< "$v"
  GROPHECY_SMINB=$mb GROPHECY_NCH=$nch GROPHECY_I2F_MAGIC=${mg:-0} python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build_v.log 2>&1 || { echo "build $v failed"; continue; }
  for rep in 1 2; do
    timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/bench_v.log 2>&1
    echo "variant $v rep $rep: $(tail -1 gpurun_out/bench_v.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]/1e9,1), "Gcand/s", round(d["ms_per_step"],3), "ms", d["best"]["index"])')"
  done
done
