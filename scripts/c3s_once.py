"""Profiling aid: one warm-up and one measured best projection of a C3s/C3h
workload (general path), for ncu -k regex:general_kernel -s 1 -c 1."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ipps_boyermk13_b200 import build as B  # noqa: E402

B.build()
from paper_conf_ipps_boyermk13_b200 import grophecy as G  # noqa: E402
from synth import records as R  # noqa: E402
from synth import skeletons as S  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3s"
c = R.config(name)
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
sp = G.Space(c["skeletons"], S.FX5600)
rec = G.synth_records(c)
for _ in range(2):
    rc, b = sp.best(pc, rec)
torch.cuda.synchronize()
print(name, rc, b.index)
