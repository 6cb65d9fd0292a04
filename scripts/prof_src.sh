#!/bin/bash
# One gpurun call: per-skeleton segment throughput + an ncu full capture (with
# source counters) of the fused best kernel on a 2^27-record C4 sample.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force --verbose > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
grep -A2 "canon_kernel" gpurun_out/build.log | grep -E "registers|spill" | head -4

timeout 900 ncu --set full --clock-control none --import-source on -k regex:canon_kernel -s 3 -c 1 -o gpurun_out/src_full -f python bench.py --n ${PROF_N:-134217728} --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_src.log 2>&1; echo "ncu rc=$?"
python scripts/ncu_lines.py gpurun_out/src_full.ncu-rep 40 > gpurun_out/lines.txt 2>&1
python scripts/ncu_summary.py gpurun_out/src_full.ncu-rep > gpurun_out/summary.txt 2>&1
ncu -i gpurun_out/src_full.ncu-rep --page raw --csv > gpurun_out/src_raw.csv 2>/dev/null
