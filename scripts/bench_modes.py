"""Throughput of every projection entry point on the C4 workload (one GPU).

    python scripts/bench_modes.py [n_records] [reps]

One JSON line per mode: best (fused argmin), eval (SoA outputs), eval_parts
(+ time components), group_best (best transformation per projection point),
crossover (break-even iterations from the components), best over the
C3-shaped plan / strided / hull workloads, best_host (host records,
PCIe-bound).  Candidates/s from CUDA events (or the
host clock for the synchronous calls), algorithmic HBM bytes per candidate,
and the fraction of MEASURED_PEAKS.json's HBM bandwidth.
"""
import json
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


def hbm_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    return json.load(open(p))["hbm_gbs"] if os.path.exists(p) else 6650.0


def timed(fn, reps, events=True):
    fn()
    torch.cuda.synchronize()
    if events:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps * 1e-3
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


def latency(pc, reps=200):
    """Per-query time of small batches (C1: 16 records, C2: 10^6): the fused
    best into device memory (CUDA events, back to back) and the synchronous
    grophecy_best (host clock, result on the host)."""
    out = torch.empty(6, dtype=torch.int64, device="cuda")
    for wname in ("c1", "c2"):
        wc = R.config(wname)
        wsp = G.Space(wc["skeletons"], S.FX5600)
        wrec = G.synth_records(wc)
        wb = wrec.batch()
        sec = timed(lambda: wsp.best_async(pc, wb, out), reps, True)
        sec_sync = timed(lambda: wsp.best(pc, wrec), reps, False)
        print(json.dumps({"mode": "latency", "workload": wname, "n": wrec.n,
                          "us_per_query_async": sec * 1e6, "us_per_query_sync": sec_sync * 1e6,
                          "cand_per_s": wrec.n / sec,
                          "launches_per_query": None}), flush=True)
        wsp.close()


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 27
    if os.environ.get("LATENCY_ONLY"):
        latency(G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)))
        return
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    cfg = R.config("c4")
    space = G.Space(cfg["skeletons"], S.FX5600)
    pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
    # an evenly spread sample of the 10^9 sweep: 16 slices (every skeleton)
    per = n // 16
    recs = [G.synth_records(cfg, k * (cfg["n"] // 16), per) for k in range(16)]
    rec = G.Records(*[torch.cat([getattr(r, f) for r in recs]) for f in ("skx", "nx", "ny", "iters")])
    n = rec.n
    peak = hbm_peak()
    out = torch.empty(6, dtype=torch.int64, device="cuda")
    h = torch.empty(n, dtype=torch.int64, device="cuda")
    d = torch.empty(n, dtype=torch.int64, device="cuda")
    t = torch.empty(n, dtype=torch.float64, device="cuda")
    parts = [torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(4)]
    # eval_parts fills them (t_iter, t_once, t_h2d, t_d2h) for the crossover line
    b = rec.batch()
    gout = torch.empty((n // 8) * 6, dtype=torch.int64, device="cuda")
    P = G.Parts(*[x.data_ptr() for x in parts])
    import ctypes as C
    st = torch.cuda.current_stream().cuda_stream
    modes = {
        "best": (lambda: space.best_async(pc, b, out), 16, True),
        "eval": (lambda: G.lib().grophecy_eval(space.h, C.byref(pc), C.byref(b), h.data_ptr(),
                                               d.data_ptr(), t.data_ptr(), C.c_void_p(st)), 40, True),
        "eval_parts": (lambda: G.lib().grophecy_eval_parts(space.h, C.byref(pc), C.byref(b),
                                                           h.data_ptr(), d.data_ptr(), t.data_ptr(),
                                                           C.byref(P), C.c_void_p(st)), 72, True),
        "group_best": (lambda: space.group_best(pc, rec, capacity=n // 8, out=gout, as_tensor=True),
                       16 + 24 + 24 + 16, False),
    }
    for name, (fn, bpc, ev) in modes.items():
        sec = timed(fn, reps, ev)
        gbs = bpc * n / sec / 1e9
        print(json.dumps({"mode": name, "n": n, "cand_per_s": n / sec, "ms": sec * 1e3,
                          "bytes_per_candidate": bpc, "hbm_GBps": gbs, "hbm_frac": gbs / peak,
                          "timer": "cuda events" if ev else "host clock (synchronous call)"}),
              flush=True)
    # layouts other than the generator's: (1) the transformations of every
    # design point in reverse order (still a sweep: any fixed order inside
    # the design points), (2) the records of consecutive design point pairs
    # interleaved, so no CTA tile is a sweep tile and everything takes the
    # general (pass-2) path
    layouts = {
        "best_reversed_xforms": lambda i: (i // 16) * 16 + 15 - (i % 16),
        "best_general_path": lambda i: (i // 32) * 32 + (i % 2) * 16 + (i % 32) // 2,
    }
    for lname, perm in layouts.items():
        idx = perm(torch.arange(n, device="cuda"))
        grec = G.Records(*[getattr(rec, f)[idx].contiguous() for f in ("skx", "nx", "ny", "iters")])
        gb = grec.batch()
        sec = timed(lambda: space.best_async(pc, gb, out), reps, True)
        gbs = 16 * n / sec / 1e9
        print(json.dumps({"mode": lname, "n": n, "cand_per_s": n / sec,
                          "ms": sec * 1e3, "bytes_per_candidate": 16, "hbm_GBps": gbs,
                          "hbm_frac": gbs / peak, "timer": "cuda events"}), flush=True)
    del grec, gb, idx
    # spaces of skeletons with 8 / 4 transformations: the sweep's design
    # points have that size (sweep_kernel<.., 8 / 4>)
    for X in (8, 4):
        xc = dict(cfg)
        xc["skeletons"] = [dict(sk, kx=sk["kx"][:X]) for sk in cfg["skeletons"]]
        xc["n_xforms"] = X
        xsp = G.Space(xc["skeletons"], S.FX5600)
        xrec = G.synth_records(dict(xc, n=n))
        xb = xrec.batch()
        sec = timed(lambda: xsp.best_async(pc, xb, out), reps, True)
        gbs = 16 * n / sec / 1e9
        print(json.dumps({"mode": f"best_x{X}", "n": n, "cand_per_s": n / sec,
                          "ms": sec * 1e3, "bytes_per_candidate": 16, "hbm_GBps": gbs,
                          "hbm_frac": gbs / peak, "timer": "cuda events"}), flush=True)
        xsp.close()
        del xrec, xb
    # next-row workloads: crossover (NEXT-2) on eval_parts outputs
    ti, to, th, td = parts
    sec = timed(lambda: G.crossover(ti, to, th, td, 1e-3), reps, True)
    gbs = 48 * n / sec / 1e9
    print(json.dumps({"mode": "crossover", "n": n, "cand_per_s": n / sec, "ms": sec * 1e3,
                      "bytes_per_candidate": 48, "hbm_GBps": gbs, "hbm_frac": gbs / peak,
                      "timer": "cuda events"}), flush=True)
    # C3-shaped workloads over the general paths (10^7 candidates, fused best):
    # plans (c3), strided sections + may-writes (c3s), hull mode (c3h)
    for wname in ("c3", "c3s", "c3h"):
        wc = R.config(wname)
        wsp = G.Space(wc["skeletons"], S.FX5600)
        wrec = G.synth_records(wc)
        wb = wrec.batch()
        sec = timed(lambda: wsp.best_async(pc, wb, out), reps, True)
        gbs = 16 * wrec.n / sec / 1e9
        print(json.dumps({"mode": "best", "workload": wname, "n": wrec.n,
                          "cand_per_s": wrec.n / sec, "ms": sec * 1e3, "bytes_per_candidate": 16,
                          "hbm_GBps": gbs, "hbm_frac": gbs / peak, "timer": "cuda events"}),
              flush=True)
        wsp.close()
        del wrec
    host = {k: getattr(rec, k).cpu().pin_memory() for k in ("skx", "nx", "ny", "iters")}
    sec = timed(lambda: space.best_host(pc, host), max(1, reps // 2), False)
    print(json.dumps({"mode": "best_host", "n": n, "cand_per_s": n / sec, "ms": sec * 1e3,
                      "h2d_bytes": 16 * n, "link_GBps": 16 * n / sec / 1e9,
                      "timer": "host clock"}), flush=True)


if __name__ == "__main__":
    main()
