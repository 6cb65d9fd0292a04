#!/bin/bash
# One gpurun call for an optimisation iteration: build, GPU tests (optional),
# bench line, ncu capture of the pass-1 kernel + phase grouping.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -z "$NO_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/pytest_gpu.log
fi
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-200
if [ -z "$NO_NCU" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-sweep_kernel} -s 3 -c 1 -o gpurun_out/${TAG:-it}_full -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
python scripts/ncu_summary.py gpurun_out/${TAG:-it}_full.ncu-rep > gpurun_out/${TAG:-it}_summary.txt 2>&1
fi
