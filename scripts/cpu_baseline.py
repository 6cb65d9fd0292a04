#!/usr/bin/env python
"""CPU baseline of SURVEY.md §8(d) on the host it runs on (the GPU box):
the oracle, as it stands, over C1, C2 and C3 in full on all cores, the same
records on one thread (C1, C2 in full; C3 on every 16th record, stated), and
C4 on a bounded 16-slice sample; the CPU model from /proc/cpuinfo.  Writes
JSON (argv[1]).  Test infrastructure: oracle/ + synth/ only.

Paper context: the applications' CPU versions ran OpenMP on 8 threads of a
Xeon E5405; the paper never timed GROPHECY++ itself.
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import oracle as O      # noqa: E402
from synth import records as R      # noqa: E402
from synth import skeletons as S    # noqa: E402


def cpu_model():
    for ln in open("/proc/cpuinfo"):
        if ln.startswith("model name"):
            return ln.split(":", 1)[1].strip()
    return None


def timed_best(P, rec, threads):
    t0 = time.perf_counter()
    rc, b = P.best(rec, nthreads=threads)
    return time.perf_counter() - t0, b


def main():
    out = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/cpu_baseline.json"
    cores = len(os.sched_getaffinity(0))
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    doc = {"cpu_model": cpu_model(), "cores": cores, "kind": "oracle (oracle/oracle.c, -O2, pthreads)",
           "configs": {}}
    for name, one_stride in (("c1", 1), ("c2", 1), ("c3", 16)):
        cfg = R.config(name)
        rec = R.gen_records(cfg)
        P = O.Problem(cfg["skeletons"], S.FX5600, link)
        dt_all, b = timed_best(P, rec, cores)
        sub = {k: v[::one_stride] for k, v in rec.items()}
        dt_one, _ = timed_best(P, sub, 1)
        doc["configs"][name] = {
            "n": cfg["n"], "best_index": int(b.index),
            "all_cores": {"seconds": dt_all, "candidates_per_s": cfg["n"] / dt_all},
            "one_thread": {"seconds": dt_one, "records": len(sub["skx"]),
                           "candidates_per_s": len(sub["skx"]) / dt_one,
                           "sample": "full" if one_stride == 1 else f"every {one_stride}th record"}}
        print(name, doc["configs"][name], flush=True)
    cfg = R.config("c4")
    per = 1 << 18
    idx = np.concatenate([np.arange(k * cfg["n"] // 16, k * cfg["n"] // 16 + per, dtype=np.uint64)
                          for k in range(16)])
    rec = R.gen_records_at(cfg, idx)
    P = O.Problem(cfg["skeletons"], S.FX5600, link)
    dt_all, _ = timed_best(P, rec, cores)
    sub = {k: v[::16] for k, v in rec.items()}
    dt_one, _ = timed_best(P, sub, 1)
    doc["configs"]["c4"] = {"n": cfg["n"], "sample": f"16 slices of {per} records at k*N/16",
                            "all_cores": {"seconds": dt_all, "candidates_per_s": len(idx) / dt_all},
                            "one_thread": {"seconds": dt_one, "records": len(sub["skx"]),
                                           "candidates_per_s": len(sub["skx"]) / dt_one,
                                           "sample": "every 16th record of the sample"}}
    print("c4", doc["configs"]["c4"], flush=True)
    os.makedirs(os.path.dirname(out) or ".", exist_ok=True)
    json.dump(doc, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
