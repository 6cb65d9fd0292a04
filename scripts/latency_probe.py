"""Per-query latency of small best projections (CUDA events, back to back):
C2 (10^6 records, 3 skeletons), C2 with one skeleton (no skeleton boundary
inside a CTA tile, so nothing is listed for pass 2), a single tile, C1."""
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


def lat(space, pc, rec, reps=300):
    out = torch.empty(6, dtype=torch.int64, device="cuda")
    b = rec.batch()
    for _ in range(20):
        space.best_async(pc, b, out)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        space.best_async(pc, b, out)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / reps


pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
c2 = R.config("c2")
one = dict(c2, skeletons=c2["skeletons"][:1], rules=c2["rules"][:1])
for name, cfg, n in (("c2", c2, 10**6), ("c2_tile_aligned", c2, 3 * 81 * 4096),
                     ("c2_one_skeleton", one, 10**6), ("c2_one_tile", one, 4096),
                     ("c2_37_tiles", one, 37 * 4096), ("c1", R.config("c1"), 16)):
    sp = G.Space(cfg["skeletons"], S.FX5600)
    rec = G.synth_records(dict(cfg, n=n))
    print(f"{name:18s} n={n:8d} {lat(sp, pc, rec):7.2f} us/query", flush=True)
    sp.close()
