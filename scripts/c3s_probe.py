"""Best projection of a C3s (strided sections) or C3h prefix: the general
path's strided / hull usage sweep, for profiling.  usage: c3s_probe.py [name] [n]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ipps_boyermk13_b200 import build  # noqa: E402

build.build()
from paper_conf_ipps_boyermk13_b200 import grophecy as G  # noqa: E402
from synth import records as R  # noqa: E402
from synth import skeletons as S  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3s"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 10**7
cfg = R.config(name)
cfg = dict(cfg, n=max(cfg["n"], n))   # (the same recipe at a larger size)
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
space = G.Space(cfg["skeletons"], S.FX5600)
rec = G.synth_records(cfg, 0, n)
out = torch.empty(6, dtype=torch.int64, device="cuda")
b = rec.batch()
space.best_async(pc, b, out)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
space.best_async(pc, b, out)
e1.record()
torch.cuda.synchronize()
print(f"{name}: {n / (e0.elapsed_time(e1) * 1e-3):.3e} cand/s")
