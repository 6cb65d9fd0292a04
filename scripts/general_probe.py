"""Best projection of 2^24 C4 records whose design points are interleaved
record by record (no sweep tile: everything runs on the general pass-2
path), for profiling the general path.  usage: general_probe.py [reps]"""
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

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
n = 1 << 24
cfg = R.config("c4")
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
space = G.Space(cfg["skeletons"], S.FX5600)
rec = G.synth_records(cfg, 0, n)
i = torch.arange(n, device="cuda")
idx = (i // 32) * 32 + (i % 2) * 16 + (i % 32) // 2
grec = G.Records(*[getattr(rec, f)[idx].contiguous() for f in ("skx", "nx", "ny", "iters")])
out = torch.empty(6, dtype=torch.int64, device="cuda")
b = grec.batch()
for _ in range(reps):
    space.best_async(pc, b, out)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
space.best_async(pc, b, out)
e1.record()
torch.cuda.synchronize()
print(f"general path: {n / (e0.elapsed_time(e1) * 1e-3):.3e} cand/s")
