#!/bin/bash
# One gpurun call: ncu full capture of the sweep kernel in the bench configuration.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-sweep_kernel} -s ${SKIP:-3} -c 1 -o gpurun_out/${TAG:-sweep}_full -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
python scripts/ncu_summary.py gpurun_out/${TAG:-sweep}_full.ncu-rep > gpurun_out/${TAG:-sweep}_summary.txt 2>&1; head -40 gpurun_out/${TAG:-sweep}_summary.txt
