#!/usr/bin/env python
"""Full-size oracle goldens for C2, C3 (and C3s/C3h) and C4 — TEST INFRASTRUCTURE.

Imports only ``oracle/`` and ``synth/`` (never the product package): every
value written here is the CPU oracle's.  Output ``tests/golden/<cfg>_full.json``:

    {"config", "n", "shards": [{"lo", "hi", <summary>}...], "total": <summary>}

with, per record range, the order-independent summary the GPU tests compare
against:

    best_index, best_t_bits   argmin of (t, global index) over valid, finite t
                              (P:L67 / P:L123: "best achievable performance";
                              N7: ties -> lowest global index)
    best_h2d, best_d2h        the best candidate's bytes
    n_valid, n_invalid, n_inf record counts (invalid -> NaN, infeasible -> +inf)
    sum_h2d, sum_d2h          sum of bytes mod 2^64 over every record
    xor_t_bits, sum_t_bits    XOR / sum mod 2^64 of the binary64 bit pattern of t
                              over the valid records (NaN excluded)

Resumable: a shard already present in the output file is skipped, so the
10^9-record C4 run (about an hour on 8 cores) may be interrupted and restarted.

    python scripts/oracle_golden.py c3            # 1 shard
    python scripts/oracle_golden.py c4 --shards 16
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from oracle import oracle as O           # noqa: E402
from synth import records as R           # noqa: E402
from synth import skeletons as S         # noqa: E402

M64 = (1 << 64) - 1


def empty_summary():
    return {"best_index": None, "best_t_bits": None, "best_h2d": None, "best_d2h": None,
            "n_valid": 0, "n_invalid": 0, "n_inf": 0, "sum_h2d": 0, "sum_d2h": 0,
            "xor_t_bits": 0, "sum_t_bits": 0}


def better(t_a, i_a, t_b, i_b):
    """(t_a, i_a) < (t_b, i_b) lexicographically; None = no candidate."""
    if t_b is None:
        return True
    return t_a < t_b or (t_a == t_b and i_a < i_b)


def fold(acc, part):
    """Merge two summaries (order-independent)."""
    out = dict(acc)
    for k in ("n_valid", "n_invalid", "n_inf"):
        out[k] = acc[k] + part[k]
    for k in ("sum_h2d", "sum_d2h", "sum_t_bits"):
        out[k] = (acc[k] + part[k]) & M64
    out["xor_t_bits"] = acc["xor_t_bits"] ^ part["xor_t_bits"]
    if part["best_index"] is not None:
        ta = None if acc["best_t_bits"] is None else float(
            np.array([acc["best_t_bits"]], np.uint64).view(np.float64)[0])
        tb = float(np.array([part["best_t_bits"]], np.uint64).view(np.float64)[0])
        if better(tb, part["best_index"], ta, acc["best_index"]):
            for k in ("best_index", "best_t_bits", "best_h2d", "best_d2h"):
                out[k] = part[k]
    return out


def summarise(h, d, t, base):
    s = empty_summary()
    valid = ~np.isnan(t)
    finite = np.isfinite(t)
    s["n_valid"] = int(valid.sum())
    s["n_invalid"] = int((~valid).sum())
    s["n_inf"] = int((valid & ~finite).sum())
    s["sum_h2d"] = int(h.sum(dtype=np.uint64)) & M64
    s["sum_d2h"] = int(d.sum(dtype=np.uint64)) & M64
    bits = t.view(np.uint64)[valid]
    s["xor_t_bits"] = int(np.bitwise_xor.reduce(bits)) if bits.size else 0
    s["sum_t_bits"] = int(bits.sum(dtype=np.uint64)) & M64
    if finite.any():
        tf = np.where(finite, t, np.inf)
        k = int(np.argmin(tf))          # first occurrence = lowest index on ties
        s["best_index"] = base + k
        s["best_t_bits"] = int(t[k:k + 1].view(np.uint64)[0])
        s["best_h2d"] = int(h[k])
        s["best_d2h"] = int(d[k])
    return s


def run(name, shards, chunk, threads, out_path, n=None):
    cfg = R.config(name)
    if n:
        cfg = R.with_n(cfg, n)
    N = cfg["n"]
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    assert rc == 0
    P = O.Problem(cfg["skeletons"], S.FX5600, link)
    doc = {"config": name, "n": N, "shards": [], "total": None,
           "source": "scripts/oracle_golden.py (oracle/ + synth/ only)",
           "pcie": "fit(1e-5, 0.2147483648, 2^29) both directions", "gpu": "FX5600"}
    if os.path.exists(out_path):
        old = json.load(open(out_path))
        if old.get("n") == N and old.get("config") == name:
            doc["shards"] = old["shards"]
    done = {(s["lo"], s["hi"]) for s in doc["shards"]}
    for r in range(shards):
        lo, hi = N * r // shards, N * (r + 1) // shards
        if (lo, hi) in done:
            continue
        t0 = time.time()
        acc = empty_summary()
        for s in range(lo, hi, chunk):
            e = min(hi, s + chunk)
            rec = R.gen_records(cfg, s, e)
            h, d, t = P.eval(rec, nthreads=threads)
            acc = fold(acc, summarise(h, d, t, s))
        acc.update({"lo": lo, "hi": hi})
        doc["shards"].append(acc)
        doc["shards"].sort(key=lambda x: x["lo"])
        with open(out_path + ".tmp", "w") as f:
            json.dump(doc, f, indent=1)
        os.replace(out_path + ".tmp", out_path)
        print(f"{name} shard {r}/{shards} [{lo},{hi}) {time.time() - t0:.1f}s "
              f"best={acc['best_index']}", flush=True)
    if len(doc["shards"]) == shards:
        tot = empty_summary()
        for s in doc["shards"]:
            tot = fold(tot, s)
        doc["total"] = tot
        with open(out_path + ".tmp", "w") as f:
            json.dump(doc, f, indent=1)
        os.replace(out_path + ".tmp", out_path)
        print(f"{name} total best={tot['best_index']} n_valid={tot['n_valid']}", flush=True)
    return doc


def main():
    p = argparse.ArgumentParser()
    p.add_argument("config")
    p.add_argument("--shards", type=int, default=1)
    p.add_argument("--chunk", type=int, default=1 << 22)
    p.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    p.add_argument("--n", type=int, default=None)
    p.add_argument("--out", default=None)
    a = p.parse_args()
    out = a.out or os.path.join(ROOT, "tests", "golden", f"{a.config}_full.json")
    run(a.config, a.shards, a.chunk, a.threads, out, a.n)


if __name__ == "__main__":
    main()
