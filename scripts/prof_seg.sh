#!/bin/bash
# One gpurun call: ncu full capture (source counters) of the pass-1 kernel on
# one skeleton segment (SEG_ONLY=<index>) of C4.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
SEG_N=${SEG_N:-8388608} timeout 600 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-canon_kernel} -s 1 -c 1 -o gpurun_out/seg_full -f python scripts/segbench.py c4 1 > gpurun_out/ncu_seg.log 2>&1; echo "ncu rc=$?"
python scripts/ncu_lines.py gpurun_out/seg_full.ncu-rep 40 > gpurun_out/seg_lines.txt 2>&1
python scripts/ncu_summary.py gpurun_out/seg_full.ncu-rep > gpurun_out/seg_summary.txt 2>&1
