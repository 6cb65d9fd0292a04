#!/bin/bash
# One gpurun call: pipe-peak microbenchmark, CPU baseline (oracle on the
# host), PCIe calibration/validation (config 5), bench line.  -> gpurun_out/
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/peaks scripts/micro/peaks.cu && timeout 120 /tmp/peaks > gpurun_out/peaks.json; echo "peaks rc=$?"; cat gpurun_out/peaks.json
if [ -z "$NO_CPU" ]; then timeout 900 python scripts/cpu_baseline.py gpurun_out/cpu_baseline.json > gpurun_out/cpu_baseline.log 2>&1; echo "cpu rc=$?"; tail -4 gpurun_out/cpu_baseline.log | cut -c1-300; fi
if [ -z "$NO_PCIE" ]; then timeout 900 python scripts/pcie_validate.py gpurun_out/pcie.json > gpurun_out/pcie.log 2>&1; echo "pcie rc=$?"; tail -6 gpurun_out/pcie.log; fi
cp gpurun_out/peaks.json profiles/peaks.json 2>/dev/null
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-300
