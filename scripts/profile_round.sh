#!/bin/bash
# One gpurun call: bench line, ncu launch list, ncu full capture of the best
# kernel in the bench configuration, PCIe validation (config 5).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench.log | cut -c1-400
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 3 -c 1 -o gpurun_out/best_full -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
if [ -z "$NO_PCIE" ]; then timeout 900 python scripts/pcie_validate.py gpurun_out/pcie.json > gpurun_out/pcie.log 2>&1; echo "pcie rc=$?"; cat gpurun_out/pcie.log | tail -4; fi
python scripts/ncu_lines.py gpurun_out/best_full.ncu-rep 40 > gpurun_out/best_lines.txt 2>&1
python scripts/ncu_summary.py gpurun_out/best_full.ncu-rep > gpurun_out/best_summary.txt 2>&1
python scripts/ncu_groups.py gpurun_out/best_full.ncu-rep > gpurun_out/best_groups.txt 2>&1
