#!/bin/bash
# A/B of the library at a git revision (ab_rev.tar: `git archive REV`) against the working
# tree: both built in-tree, benched alternately (C4, N = 1).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
cp paper_conf_ipps_boyermk13_b200/libgrophecy.so /tmp/lib_b.so
if [ -d /tmp/ab_rev ]; then rm -rf /tmp/ab_rev; fi
mkdir -p /tmp/ab_rev && tar -C /tmp/ab_rev -xf ab_rev.tar
( cd /tmp/ab_rev && python -m paper_conf_ipps_boyermk13_b200.build --force > /dev/null 2>&1 ) && cp /tmp/ab_rev/paper_conf_ipps_boyermk13_b200/libgrophecy.so /tmp/lib_a.so
for r in 1 2 3; do
  for v in a b; do
    echo "$v: $(GROPHECY_LIB=/tmp/lib_$v.so timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]/1e9,1))')"
  done
done
