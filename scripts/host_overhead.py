"""Host-side cost of one best_async call (Python ctypes marshalling + the C
launch path) vs the per-query time of back-to-back C2 queries."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ipps_boyermk13_b200 import build  # noqa: E402

build.build()
from paper_conf_ipps_boyermk13_b200 import grophecy as G  # noqa: E402
from synth import records as R  # noqa: E402
from synth import skeletons as S  # noqa: E402

pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
c = R.config("c2")
sp = G.Space(c["skeletons"], S.FX5600)
rec = G.synth_records(c)
b = rec.batch()
out = torch.empty(6, dtype=torch.int64, device="cuda")
for _ in range(50):
    sp.best_async(pc, b, out)
torch.cuda.synchronize()
n = 400
t0 = time.perf_counter()
for _ in range(n):
    sp.best_async(pc, b, out)
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
print(f"host enqueue {1e6 * (t1 - t0) / n:.2f} us/call; enqueue+drain {1e6 * (t2 - t0) / n:.2f} us/query")
