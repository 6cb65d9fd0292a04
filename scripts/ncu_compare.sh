#!/bin/bash
# ncu full captures of the sweep kernel for build variants (VARIANTS as in
# phase_timing.sh), summaries in gpurun_out/cmp_<i>_summary.txt.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
i=0
for v in ${VARIANTS:--}; do
  envs=""; [ "$v" != "-" ] && envs=$(echo "$v" | tr ',' ' ')
  env $envs python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || tail gpurun_out/build.log
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 3 -c 1 -o gpurun_out/cmp_$i -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$i.log 2>&1; echo "variant $v -> cmp_$i rc=$?"
  python scripts/ncu_summary.py gpurun_out/cmp_$i.ncu-rep > gpurun_out/cmp_${i}_summary.txt 2>&1
  i=$((i+1))
done
