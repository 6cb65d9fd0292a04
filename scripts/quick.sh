#!/bin/bash
# One gpurun call: build, GPU tests, per-skeleton segment throughput.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force --verbose > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout ${PYTEST_TIMEOUT:-1200} python -m pytest tests -m gpu -x -q --timeout 900 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
timeout 600 python scripts/segbench.py ${SEG_CFG:-c4} 5 > gpurun_out/seg.txt 2>&1; cat gpurun_out/seg.txt | cut -c1-200
