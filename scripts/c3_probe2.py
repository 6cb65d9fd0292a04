"""C3 overhead probe: 10^7 records with 64 skeletons (the config), with 8 and
with 1 skeleton (fewer boundaries / table changes), and 10^8 records."""
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

pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
c3 = R.config("c3")
out = torch.empty(6, dtype=torch.int64, device="cuda")
for k, n in ((64, 10**7), (8, 10**7), (1, 10**7), (64, 10**8)):
    cfg = dict(c3, skeletons=c3["skeletons"][:k], rules=c3["rules"][:k], n=n)
    sp = G.Space(cfg["skeletons"], S.FX5600)
    rec = G.synth_records(cfg)
    b = rec.batch()
    for _ in range(3):
        sp.best_async(pc, b, out)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        sp.best_async(pc, b, out)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    print(f"skeletons={k:3d} n={n:10d} {ms*1e3:8.1f} us  {n / (ms * 1e-3):.3e} cand/s", flush=True)
    sp.close()
