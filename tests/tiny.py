"""Random tiny skeletons for brute-force property tests (test helper).

Extents at the chosen (nx, ny) stay <= 24 x 24 so the literal per-element
bitmap is cheap.  Boxes include empty, inverted, negative and out-of-range
bounds; modes R / W / RW; whole-array reads; live-out on/off.
"""
import numpy as np


DUMMY_KX = {"tpb": 64, "ipt": 1, "regs": 8, "smem": 0, "total": 10.0, "coal": 1.0,
            "uncoal": 0.0, "upm": 32.0, "lbpw": 128.0, "synch": 0.0}


def _a8_const(v):
    return (int(v), 0, 0, 0)


def random_tiny_skeleton(rng, n_xforms=1, max_kernels=8, max_arrays=3, max_regions=12,
                         strided=False, maywrite=False, hull=False, rank3=False):
    """strided: BRS strides in {1, 2, 3, 4, 6} per dimension (lcm <= 12);
    maywrite: irregular (WHOLE) writes too; hull: the approximate-UNION mode;
    rank3: arrays get 1-5 (possibly size-dependent) planes and regions plane
    ranges (N4r)."""
    nx = int(rng.integers(1, 13))
    ny = int(rng.integers(1, 13))
    n_arr = int(rng.integers(1, max_arrays + 1))
    arrays = []
    for _ in range(n_arr):
        # extents that depend on (nx, ny): rows = ny + r, cols = 2*nx - c, etc.
        kind = int(rng.integers(0, 3))
        if kind == 0:
            rows, cols = (int(rng.integers(0, 4)), 0, 8, 0), (int(rng.integers(-1, 4)), 8, 0, 0)
        elif kind == 1:
            rows, cols = (1, 0, 0, 0), (int(rng.integers(0, 3)), 0, 0, 8)   # 1-D nx*ny
        else:
            rows, cols = _a8_const(rng.integers(0, 9)), (0, 16, 0, 0)
        arrays.append({"name": "a", "rows": rows, "cols": cols,
                       "elem_bytes": int(rng.choice([1, 4, 8, 16])),
                       "liveout": bool(rng.integers(0, 2))})
        if rank3:
            arrays[-1]["planes"] = ((int(rng.integers(1, 6)), 0, 0, 0) if rng.random() < 0.6
                                    else (int(rng.integers(0, 2)), 2, 0, 0))   # c0 + nx/4
            if kind == 1:
                arrays[-1]["rows"] = (1, 0, 0, 0)
                arrays[-1]["cols"] = (int(rng.integers(0, 3)), 8, 0, 0)   # keep P*R*C small
    K = int(rng.integers(1, max_kernels + 1))
    kernels = [{"name": f"k{k}", "work": (0, 0, 0, 8), "per_iter": True} for k in range(K)]
    regions = []
    for _ in range(int(rng.integers(0, max_regions + 1))):
        a = int(rng.integers(0, n_arr))
        mode = ["R", "W", "RW"][int(rng.integers(0, 3))]
        whole = (mode == "R" or maywrite) and rng.random() < 0.15

        def bound():
            # mix constants and size-scaled terms, some negative / too large
            c0 = int(rng.integers(-3, 10))
            c1 = int(rng.integers(-4, 9)) if rng.random() < 0.5 else 0
            c2 = int(rng.integers(-4, 9)) if rng.random() < 0.5 else 0
            return (c0, c1, c2, 0)

        reg = {"kernel": int(rng.integers(0, K)), "array": a, "mode": mode,
               "whole": bool(whole), "r0": bound(), "r1": bound(),
               "c0": bound(), "c1": bound()}
        if strided:
            reg["r_step"] = int(rng.choice([1, 1, 2, 3, 4, 6]))
            reg["c_step"] = int(rng.choice([1, 1, 2, 3, 4, 6]))
        if rank3 and rng.random() < 0.7:
            reg["p0"] = (int(rng.integers(-1, 4)), int(rng.integers(0, 3)) if rng.random() < 0.3 else 0, 0, 0)
            reg["p1"] = (int(rng.integers(0, 6)), int(rng.integers(0, 3)) if rng.random() < 0.3 else 0, 0, 0)
        regions.append(reg)
    kx = [[DUMMY_KX] * K] * n_xforms
    sk = {"name": "tiny", "arrays": arrays, "kernels": kernels, "regions": regions, "kx": kx}
    if hull:
        sk["hull"] = True
    return sk, nx, ny


def rng(seed):
    return np.random.default_rng(seed)
