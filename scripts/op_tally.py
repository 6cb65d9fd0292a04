#!/usr/bin/env python
"""Algorithmic op tally per candidate of each workload (oracle/ + synth/ only)
-> profiles/op_tally.json, read by bench.py for the op-bound roofline
(the rule is stated in oracle/oracle.c oracle_op_tally_one).

The mean over an evenly spaced sample of the workload (every skeleton's
index range is hit in proportion), usage amortised over the X = 16
transformations of a design point.

    python scripts/op_tally.py [--sample 65536]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import oracle as O      # noqa: E402
from synth import records as R      # noqa: E402
from synth import skeletons as S    # noqa: E402


def tally(name, sample):
    cfg = R.config(name)
    n = cfg["n"]
    m = min(sample, n)
    idx = (np.arange(m, dtype=np.uint64) * np.uint64(n // m)) if m < n else np.arange(n, dtype=np.uint64)
    rec = R.gen_records_at(cfg, idx)
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    P = O.Problem(cfg["skeletons"], S.FX5600, link)
    t = P.op_tally(rec, X=cfg["n_xforms"])
    t["sample"] = f"{len(idx)} records at stride {max(1, n // m)} over [0, {n})"
    return t


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sample", type=int, default=65536)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "op_tally.json"))
    a = ap.parse_args()
    doc = {"rule": "oracle/oracle.c oracle_op_tally_one (DESIGN.md §6): fp64 ops (division by a "
                   "space constant = 2), int ops, int->fp64 conversions per candidate; "
                   "size-independent work amortised per space, usage per design point",
           "source": "scripts/op_tally.py (oracle/ + synth/ only)"}
    for name in ("c1", "c2", "c3", "c4"):
        doc[name] = tally(name, a.sample)
        print(name, doc[name], flush=True)
    json.dump(doc, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
