"""Candidate records and the five BASELINE.json configurations.

Record i (global index) of a config with N records, X transformations per
group, S skeletons:

    g     = i // X                 (group: one (skeleton, size, iters) point)
    xform = i %  X
    G     = ceil(N / X)
    skel  = (g * S) // G           (skeleton-major contiguous ranges)
    z_j   = splitmix.counter(seed, 4*g + j),  j = 0, 1, 2
    size rule of skel:
        "square": n = lo + z_0 % (hi-lo+1);  nx = ny = n
        "indep" : nx = lo + z_0 % span;  ny = lo + z_1 % span
        "oned"  : nx = lo + z_0 % span;  ny = 1
        "fixed" : nx, ny = lo, hi
    iters = it_lo + z_2 % (it_hi - it_lo + 1)

SoA layout: four uint32 arrays skx = (skel << 16) | xform, nx, ny, iters.
The CUDA generator (grophecy_synth_records) implements this independently.
"""
import numpy as np

from . import skeletons as sk
from .splitmix import counter

# size-rule kinds (shared integer codes with the CUDA generator's table)
SQUARE, INDEP, ONED, FIXED = 0, 1, 2, 3


def make_rule(kind, lo, hi, it_lo=1, it_hi=1024):
    return {"kind": kind, "lo": lo, "hi": hi, "it_lo": it_lo, "it_hi": it_hi}


def gen_records(cfg, start=0, stop=None):
    """Records [start, stop) of config ``cfg`` as four uint32 numpy arrays."""
    if stop is None:
        stop = cfg["n"]
    return gen_records_at(cfg, np.arange(start, stop, dtype=np.uint64))


def gen_records_at(cfg, i):
    """Records at arbitrary global indices ``i`` (uint64 array)."""
    N, X, seed, rules = cfg["n"], cfg["n_xforms"], cfg["seed"], cfg["rules"]
    S = len(rules)
    G = (N + X - 1) // X
    i = np.asarray(i, dtype=np.uint64)
    g = i // np.uint64(X)
    x = (i % np.uint64(X)).astype(np.uint32)
    skel = ((g * np.uint64(S)) // np.uint64(G)).astype(np.int64)
    z0 = counter(seed, g * np.uint64(4))
    z1 = counter(seed, g * np.uint64(4) + np.uint64(1))
    z2 = counter(seed, g * np.uint64(4) + np.uint64(2))
    kind = np.array([r["kind"] for r in rules], dtype=np.int64)[skel]
    lo = np.array([r["lo"] for r in rules], dtype=np.uint64)[skel]
    hi = np.array([r["hi"] for r in rules], dtype=np.uint64)[skel]
    itlo = np.array([r["it_lo"] for r in rules], dtype=np.uint64)[skel]
    ithi = np.array([r["it_hi"] for r in rules], dtype=np.uint64)[skel]
    span = hi - lo + np.uint64(1)
    span_safe = np.where(kind == FIXED, np.uint64(1), span)
    a = lo + z0 % span_safe
    b = lo + z1 % span_safe
    nx = np.where(kind == FIXED, lo, a)
    ny = np.select([kind == SQUARE, kind == INDEP, kind == ONED, kind == FIXED],
                   [a, b, np.ones_like(a), hi])
    iters = itlo + z2 % (ithi - itlo + np.uint64(1))
    skx = (skel.astype(np.uint32) << np.uint32(16)) | x
    return {"skx": skx.astype(np.uint32), "nx": nx.astype(np.uint32),
            "ny": ny.astype(np.uint32), "iters": iters.astype(np.uint32)}


def config(name):
    """Build config C1..C4 (BASELINE.json ``configs[0..3]``)."""
    if name == "c1":
        skels = [sk.s0_stencil2()]
        rules = [make_rule(FIXED, 64, 64, 1, 1)]
        return {"name": "c1", "skeletons": skels, "rules": rules, "n": 16,
                "n_xforms": 16, "seed": 0x5EED0001}
    if name == "c2":
        skels = [sk.s1_hotspot(), sk.s2_hotspot_pp2(), sk.s3_srad()]
        rules = [make_rule(SQUARE, 256, 8192)] * 3
        return {"name": "c2", "skeletons": skels, "rules": rules, "n": 10**6,
                "n_xforms": 16, "seed": 0x5EED0002}
    if name == "c3":
        skels = sk.random_skeletons(0x5EED0003, 64)
        rules = [make_rule(INDEP, 256, 8192)] * 64
        return {"name": "c3", "skeletons": skels, "rules": rules, "n": 10**7,
                "n_xforms": 16, "seed": 0x5EED0003}
    if name == "c4":
        skels = [f() for f in sk.LIBRARY] + sk.random_skeletons(0x5EED0004, 9)
        rules = []
        for s in skels:
            if s["name"] in ("cfd", "vecadd"):
                rules.append(make_rule(ONED, 1 << 10, 1 << 20))
            elif s["name"] == "stassuij":
                rules.append(make_rule(FIXED, 2048, 132))
            else:
                rules.append(make_rule(SQUARE, 256, 8192))
        return {"name": "c4", "skeletons": skels, "rules": rules, "n": 10**9,
                "n_xforms": 16, "seed": 0x5EED0004}
    if name in ("c3s", "c3h"):
        # NEXT-3 workloads (not BASELINE configs): C3's shape with strided
        # sections and irregular writes; "c3h" in the approximate hull mode
        skels = sk.random_skeletons(0x5EED0033, 64, brs=True, hull=name == "c3h")
        rules = [make_rule(INDEP, 256, 8192)] * 64
        return {"name": name, "skeletons": skels, "rules": rules, "n": 10**7,
                "n_xforms": 16, "seed": 0x5EED0033}
    raise ValueError(name)


def with_n(cfg, n):
    """Same workload recipe, different record count (parity-test sizes)."""
    out = dict(cfg)
    out["n"] = n
    return out

