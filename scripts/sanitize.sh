#!/bin/bash
# One gpurun call: compute-sanitizer memcheck / racecheck / synccheck over
# small best / eval projections (C1, a C2 prefix, a C4 prefix with several
# sweep tiles, a partial tile and the general path).
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
python -m paper_conf_ipps_boyermk13_b200.build --force > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
cat > /tmp/san_run.py <<'PY'
import sys
sys.path.insert(0, ".")
import numpy as np, torch
from paper_conf_ipps_boyermk13_b200 import grophecy as G
from synth import records as R, skeletons as S
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
for name, n in (("c1", 16), ("c2", 3 * 4096 + 16 * 9), ("c4", 5 * 4096 + 16 * 40 + 3), ("c3s", 4096)):
    c = R.config(name)
    sp = G.Space(c["skeletons"], S.FX5600)
    rec = G.synth_records(c, 0, n)
    rc, b = sp.best(pc, rec)
    sp.eval(pc, rec)
    torch.cuda.synchronize()
    print(name, n, b.index, b.n_valid)
    sp.close()
PY
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san_run.py > gpurun_out/san_$tool.log 2>&1
  echo "== $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san_$tool.log | tail -1)"
done
