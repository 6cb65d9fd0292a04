"""Skeleton library shaped like the paper's workloads.

A skeleton is a dict::

    {"name": str,
     "arrays":  [{"name", "rows": A8, "cols": A8, "elem_bytes": int, "liveout": bool}],
     "kernels": [{"name", "work": A8, "per_iter": bool}],
     "regions": [{"kernel": k, "array": a, "mode": "R"|"W"|"RW", "whole": bool,
                  "r0": A8, "r1": A8, "c0": A8, "c1": A8}],
     "kx":      [[{tpb, ipt, regs, smem, total, coal, uncoal, upm, lbpw, synch}
                  for each kernel] for each transformation]}

``A8 = (c0, c1, c2, c3)`` denotes the size-affine value
``c0 + floor((c1*nx + c2*ny + c3*nx*ny) / 8)``.  Evaluating
it is the method's job (oracle / CUDA side); this module only writes the
coefficients down.

Paper anchors: HotSpot 3x3 stencil over a grid, iterations fusable;
SRAD two kernels, coefficient arrays consumed by the update kernel;
CFD three-kernel Euler solver on an unstructured mesh, transfers independent of
the iteration count; Stassuij CSR 132x132 real times dense
132x2048 complex; vector add.  Region boxes are
"bounded regular sections"; "whole" reads model the conservative
irregular rule.
"""
from .splitmix import Stream

# ---- affine8 coefficient helpers (pure data) --------------------------------
ZERO = (0, 0, 0, 0)


def CONST(v):
    return (v, 0, 0, 0)


NX = (0, 8, 0, 0)
NY = (0, 0, 8, 0)
NXNY = (0, 0, 0, 8)


def nx_times(words):
    return (0, 8 * words, 0, 0)


def region(kernel, array, mode, arrays=None, whole=False, box=None):
    """box = (r0, r1, c0, c1) A8 tuples; full=True-style boxes come from the
    array's own extent coefficients."""
    if box is None:
        a = arrays[array]
        box = (ZERO, a["rows"], ZERO, a["cols"])
    r0, r1, c0, c1 = box
    return {"kernel": kernel, "array": array, "mode": mode, "whole": bool(whole),
            "r0": r0, "r1": r1, "c0": c0, "c1": c1}


def full(kernel, array, mode, arrays):
    """Regular access to the whole array, written as an explicit box."""
    return region(kernel, array, mode, arrays=arrays)


def whole_read(kernel, array, arrays):
    """Irregular/whole read: the GROPHECY_REGION_WHOLE flag."""
    return region(kernel, array, "R", arrays=arrays, whole=True)


INTERIOR = ((1, 0, 0, 0), (-1, 0, 8, 0), (1, 0, 0, 0), (-1, 8, 0, 0))  # [1,ny-1)x[1,nx-1)

# ---- transformation tables (SURVEY App. A "Stencil xform table X = 16") -----
TPB4 = (64, 128, 256, 512)
# v: (total, coal, uncoal, ipt, synch, regs, smem_per_tpb)  for 2 memory instrs/item
_VARIANTS = (
    (40.0, 10.0, 0.0, 1, 0, 12, 0),    # naive
    (48.0, 2.25, 0.0, 1, 1, 14, 6),    # smem tiling
    (70.0, 17.0, 0.0, 2, 0, 20, 0),    # coarse2 (2 items / thread)
    (40.0, 0.0, 10.0, 1, 0, 12, 0),    # uncoalesced
)


def stencil_kx(scale=1.0, extra=0.0):
    """16 transformations x = 4*t + v.  ``scale`` multiplies the memory/compute
    instruction counts (memory instructions per item / 2); ``extra`` adds that
    many extra memory instructions per item (coalesced for v0-v2, scaled by
    ipt; uncoalesced for v3)."""
    out = []
    for t in range(4):
        tpb = TPB4[t]
        for v in range(4):
            total, coal, uncoal, ipt, synch, regs, smem = _VARIANTS[v]
            total, coal, uncoal = total * scale, coal * scale, uncoal * scale
            if v < 3:
                coal += extra * ipt
            else:
                uncoal += extra
            out.append({"tpb": tpb, "ipt": ipt, "regs": regs, "smem": smem * tpb,
                        "total": total, "coal": coal, "uncoal": uncoal,
                        "upm": 32.0, "lbpw": 128.0, "synch": float(synch)})
    return out


def _kx_for(kernels, per_kernel):
    """per_kernel: list (one per kernel) of 16-entry lists -> [x][k] table."""
    nx_ = len(per_kernel[0])
    return [[per_kernel[k][x] for k in range(len(kernels))] for x in range(nx_)]


def _mem_scale(regions, k):
    n = sum((1 if "R" in r["mode"] else 0) + (1 if "W" in r["mode"] else 0)
            for r in regions if r["kernel"] == k)
    return n / 2.0


# ---- S0 stencil2 (C1) -------------------------------------------------------
def s0_stencil2():
    arrays = [{"name": "A", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": True},
              {"name": "B", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": False}]
    w = (4, -16, -16, 8)  # (nx-2)(ny-2)
    kernels = [{"name": "k0", "work": w, "per_iter": True},
               {"name": "k1", "work": w, "per_iter": True}]
    regions = [whole_read(0, 0, arrays), region(0, 1, "W", box=INTERIOR),
               whole_read(1, 1, arrays), region(1, 0, "W", box=INTERIOR)]
    t = stencil_kx()
    return {"name": "stencil2", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, [t, t])}


# ---- S1 hotspot ----------------------------------------------------
def s1_hotspot():
    arrays = [{"name": "temp_in", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": False},
              {"name": "power", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": False},
              {"name": "temp_out", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": True}]
    kernels = [{"name": "hotspot", "work": NXNY, "per_iter": True}]
    regions = [whole_read(0, 0, arrays), whole_read(0, 1, arrays), full(0, 2, "W", arrays)]
    t = stencil_kx(extra=1.0)
    return {"name": "hotspot", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, [t])}


# ---- S2 hotspot ping-pong, two iterations unrolled ---------------------------
def s2_hotspot_pp2():
    arrays = [{"name": "t0", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": True},
              {"name": "p", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": False},
              {"name": "t1", "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": False}]
    kernels = [{"name": "hs_even", "work": NXNY, "per_iter": True},
               {"name": "hs_odd", "work": NXNY, "per_iter": True}]
    regions = [whole_read(0, 0, arrays), whole_read(0, 1, arrays), full(0, 2, "W", arrays),
               whole_read(1, 2, arrays), whole_read(1, 1, arrays), full(1, 0, "W", arrays)]
    t = stencil_kx(extra=1.0)
    return {"name": "hotspot_pp2", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, [t, t])}


# ---- S3 srad ---------------------------------------------------------
def s3_srad():
    names = ["J", "c", "dN", "dS", "dW", "dE"]
    arrays = [{"name": n, "rows": NY, "cols": NX, "elem_bytes": 4, "liveout": n == "J"}
              for n in names]
    kernels = [{"name": "srad_coef", "work": NXNY, "per_iter": True},
               {"name": "srad_update", "work": NXNY, "per_iter": True}]
    regions = [whole_read(0, 0, arrays)] + [full(0, a, "W", arrays) for a in range(1, 6)]
    regions += [whole_read(1, a, arrays) for a in range(6)] + [full(1, 0, "W", arrays)]
    per_k = [stencil_kx(scale=_mem_scale(regions, k)) for k in range(2)]
    return {"name": "srad", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, per_k)}


# ---- S4 cfd (euler3d shape, nelr = nx, 1-D word arrays) --------
def s4_cfd():
    spec = [("variables", 5, True), ("old_variables", 5, False), ("areas", 1, False),
            ("esel", 4, False), ("normals", 12, False), ("step_factors", 1, False),
            ("fluxes", 5, False)]
    arrays = [{"name": n, "rows": CONST(1), "cols": nx_times(w), "elem_bytes": 4,
               "liveout": lo} for n, w, lo in spec]
    V, OV, AR, ES, NO, SF, FL = range(7)
    kernels = [{"name": "initialize_variables", "work": NX, "per_iter": False},
               {"name": "copy_old", "work": NX, "per_iter": True},
               {"name": "compute_step_factor", "work": NX, "per_iter": True},
               {"name": "compute_flux", "work": NX, "per_iter": True},
               {"name": "time_step", "work": NX, "per_iter": True}]
    regions = [full(0, V, "W", arrays),
               full(1, V, "R", arrays), full(1, OV, "W", arrays),
               full(2, V, "R", arrays), full(2, AR, "R", arrays), full(2, SF, "W", arrays),
               whole_read(3, V, arrays), full(3, ES, "R", arrays), full(3, NO, "R", arrays),
               full(3, FL, "W", arrays),
               full(4, OV, "R", arrays), full(4, SF, "R", arrays), full(4, FL, "R", arrays),
               full(4, V, "W", arrays)]
    per_k = [stencil_kx(scale=_mem_scale(regions, k)) for k in range(5)]
    return {"name": "cfd", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, per_k)}


# ---- S5 vector add -------------------------------------------------
def s5_vecadd():
    arrays = [{"name": n, "rows": CONST(1), "cols": NX, "elem_bytes": 4, "liveout": n == "c"}
              for n in ("a", "b", "c")]
    kernels = [{"name": "vecadd", "work": NX, "per_iter": True}]
    regions = [full(0, 0, "R", arrays), full(0, 1, "R", arrays), full(0, 2, "W", arrays)]
    per_k = [stencil_kx(scale=_mem_scale(regions, 0))]
    return {"name": "vecadd", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, per_k)}


# ---- S6 stassuij: CSR 132x132 (dense upper bound nnz=17424) x 132x2048 complex
STASSUIJ_NNZ = 132 * 132


def s6_stassuij():
    arrays = [{"name": "val", "rows": CONST(1), "cols": CONST(STASSUIJ_NNZ), "elem_bytes": 8, "liveout": False},
              {"name": "col", "rows": CONST(1), "cols": CONST(STASSUIJ_NNZ), "elem_bytes": 4, "liveout": False},
              {"name": "ptr", "rows": CONST(1), "cols": CONST(133), "elem_bytes": 4, "liveout": False},
              {"name": "B", "rows": NY, "cols": NX, "elem_bytes": 16, "liveout": False},
              {"name": "C", "rows": NY, "cols": NX, "elem_bytes": 16, "liveout": True}]
    kernels = [{"name": "csrmm", "work": NXNY, "per_iter": True}]
    regions = [whole_read(0, 0, arrays), whole_read(0, 1, arrays), whole_read(0, 2, arrays),
               whole_read(0, 3, arrays), full(0, 4, "RW", arrays)]
    per_k = [stencil_kx(scale=_mem_scale(regions, 0))]
    return {"name": "stassuij", "arrays": arrays, "kernels": kernels,
            "regions": regions, "kx": _kx_for(kernels, per_k)}


LIBRARY = [s0_stencil2, s1_hotspot, s2_hotspot_pp2, s3_srad, s4_cfd, s5_vecadd, s6_stassuij]


# ---- Generator R: random multi-kernel skeletons (C3/C4) -----------------------
def random_skeleton(st: Stream, n_xforms=16, name="R", brs=False, hull=False):
    """Generator R.  brs=True adds the full-BRS features of
    SURVEY §8(f) NEXT-3: strides in {1, 2, 3, 4} on partial boxes and
    irregular ("may") writes; hull=True marks the skeleton for the
    approximate-UNION mode.  Both only add draws, so brs=False keeps the
    original stream."""
    K = st.randint(4, 16)
    arrays = [{"name": f"a{i}", "rows": NY, "cols": NX,
               "elem_bytes": st.choice((4, 8)), "liveout": st.bernoulli(0.5)}
              for i in range(8)]
    kernels = []
    regions = []

    def access(k, a, mode):
        if st.bernoulli(0.3):
            if mode == "R":
                regions.append(whole_read(k, a, arrays))
            elif brs and st.bernoulli(0.3):
                regions.append(region(k, a, mode, arrays=arrays, whole=True))   # may-write
            else:
                regions.append(full(k, a, mode, arrays))
            return
        p0 = st.randint(0, 7)
        p1 = st.randint(p0 + 1, 8)
        q0 = st.randint(0, 7)
        q1 = st.randint(q0 + 1, 8)
        d0, d1, e0, e1 = (st.randint(0, 2) - 1 for _ in range(4))
        box = ((d0, 0, p0, 0), (d1, 0, p1, 0), (e0, q0, 0, 0), (e1, q1, 0, 0))
        reg = region(k, a, mode, box=box)
        if brs:
            reg["r_step"] = st.choice((1, 1, 2, 3, 4))
            reg["c_step"] = st.choice((1, 1, 2, 4))
        regions.append(reg)

    for k in range(K):
        q = st.randint(1, 8)
        per_iter = not (k == 0 and st.bernoulli(0.25))
        kernels.append({"name": f"k{k}", "work": (0, 0, 0, q), "per_iter": per_iter})
        for a in st.sample(8, st.randint(1, 3)):
            access(k, a, "R")
        for a in st.sample(8, st.randint(1, 2)):
            access(k, a, "W")

    kx = []
    for x in range(n_xforms):
        row = []
        for k in range(K):
            coal = float(st.randint(0, 20))
            uncoal = 0.0 if st.bernoulli(0.5) else float(st.randint(1, 10))
            total = float(st.randint(10, 200))
            if total < coal + uncoal:
                total = coal + uncoal
            smem = 0 if st.bernoulli(0.5) else st.randint(256, 16384)
            row.append({"tpb": st.choice(TPB4), "ipt": st.choice((1, 2, 4)),
                        "regs": st.randint(8, 32), "smem": smem,
                        "total": total, "coal": coal, "uncoal": uncoal,
                        "upm": 32.0, "lbpw": 128.0, "synch": float(st.randint(0, 2))})
        kx.append(row)
    out = {"name": name, "arrays": arrays, "kernels": kernels, "regions": regions, "kx": kx}
    if hull:
        out["hull"] = True
    return out


def random_skeletons(seed, count, n_xforms=16, brs=False, hull=False):
    st = Stream(seed)
    return [random_skeleton(st, n_xforms, name=f"R{seed:x}_{i}", brs=brs, hull=hull)
            for i in range(count)]


# ---- GPU model presets (CC 1.0 / Quadro FX 5600) --
FX5600 = {"n_sm": 16, "warp_size": 32, "max_threads_per_block": 512, "max_blocks_per_sm": 8,
          "max_threads_per_sm": 768, "regs_per_sm": 8192, "smem_per_sm": 16384,
          "freq_hz": 1.35e9, "mem_bw_Bps": 76.8e9, "mem_ld_cycles": 420.0,
          "dep_del_coal": 4.0, "dep_del_uncoal": 10.0, "issue_cycles": 4.0}

# The paper's PCIe magnitudes: alpha ~ 10 us, 1/beta ~ 2.5 GB/s; as
# the two measurements of P:L113: t_S = 1e-5 s, t_L = 0.2147483648 s for 2^29 B.
PAPER_TS = 1e-5
PAPER_TL = 0.2147483648
PAPER_SL = 1 << 29

# A second, modern preset (B200-class numbers) to exercise other regimes.
B200_LIKE = {"n_sm": 148, "warp_size": 32, "max_threads_per_block": 1024,
             "max_blocks_per_sm": 32, "max_threads_per_sm": 2048, "regs_per_sm": 65536,
             "smem_per_sm": 233472, "freq_hz": 1.965e9, "mem_bw_Bps": 7.7e12,
             "mem_ld_cycles": 600.0, "dep_del_coal": 4.0, "dep_del_uncoal": 20.0,
             "issue_cycles": 1.0}
