"""Per-skeleton-segment throughput of the fused best kernel (profiling aid).

    python scripts/segbench.py [config] [reps]
Prints one line per skeleton segment: candidates/s and ns/candidate.
"""
import json
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


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "c4"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    cfg = R.config(name)
    N = cfg["n"]
    ns = len(cfg["skeletons"])
    pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
    space = G.Space(cfg["skeletons"], S.FX5600)
    out = G.best_result_tensor()
    rows = []
    Gn = (N + 15) // 16
    only = os.environ.get("SEG_ONLY")
    for s in range(ns):
        if only is not None and s not in [int(v) for v in only.split(",")]:
            continue
        g0 = -(-s * Gn // ns)
        g1 = -(-(s + 1) * Gn // ns)
        lo, hi = g0 * 16, min(N, g1 * 16)
        m = min(hi - lo, int(os.environ.get("SEG_N", 1 << 25)))
        rec = G.synth_records(cfg, lo, m)
        b = rec.batch(index_base=lo)
        space.best_async(pc, b, out)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            space.best_async(pc, b, out)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        sk = cfg["skeletons"][s]
        rows.append({"skel": s, "name": sk["name"], "kernels": len(sk["kernels"]),
                     "arrays": len(sk["arrays"]), "regions": len(sk["regions"]),
                     "n": m, "cand_per_s": m / (ms * 1e-3), "ns_per_cand": ms * 1e6 / m})
        del rec
    for r in rows:
        print(json.dumps(r))
    tot = sum(r["ns_per_cand"] for r in rows) / len(rows)
    print(json.dumps({"mean_ns_per_cand": tot, "cand_per_s": 1e9 / tot}))


if __name__ == "__main__":
    main()
