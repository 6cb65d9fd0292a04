#!/bin/bash
# One gpurun call: ncu full captures (source counters) of the pass-1 kernel on
# the C4 skeleton segments listed in SEGS (default "1 8").
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for s in ${SEGS:-1 8}; do
  SEG_ONLY=$s SEG_N=${SEG_N:-8388608} timeout 600 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-canon_kernel} -s 1 -c 1 -o gpurun_out/seg${s}_full -f python scripts/segbench.py c4 1 > gpurun_out/ncu_seg$s.log 2>&1; echo "seg $s ncu rc=$?"
  python scripts/ncu_lines.py gpurun_out/seg${s}_full.ncu-rep 30 > gpurun_out/seg${s}_lines.txt 2>&1
  python scripts/ncu_summary.py gpurun_out/seg${s}_full.ncu-rep > gpurun_out/seg${s}_summary.txt 2>&1
  ncu -i gpurun_out/seg${s}_full.ncu-rep --page raw --csv > gpurun_out/seg${s}_raw.csv 2>/dev/null
done
