"""ctypes loader for the C oracle — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
``--impl reference``) may import this module.  It marshals the neutral
skeleton dicts from ``synth`` into the oracle's own structs (oracle.h);
nothing here is shared with the product package.
"""
import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liboracle.so")


def build(force=False):
    src = [os.path.join(HERE, "oracle.c"), os.path.join(HERE, "oracle.h")]
    if not force and os.path.exists(LIB_PATH) and all(
            os.path.getmtime(LIB_PATH) >= os.path.getmtime(s) for s in src):
        return LIB_PATH
    cmd = ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
           "-shared", "-pthread", "-Wall", "-Wextra", "-o", LIB_PATH, src[0], "-lm"]
    subprocess.check_call(cmd)
    return LIB_PATH


class Affine8(C.Structure):
    _fields_ = [("c0", C.c_int32), ("c1", C.c_int32), ("c2", C.c_int32), ("c3", C.c_int32)]


class Array(C.Structure):
    _fields_ = [("rows", Affine8), ("cols", Affine8), ("elem_bytes", C.c_uint32),
                ("liveout", C.c_uint32), ("planes", Affine8)]


class Region(C.Structure):
    _fields_ = [("kernel", C.c_uint32), ("array", C.c_uint32), ("mode", C.c_uint32),
                ("whole", C.c_uint32), ("r0", Affine8), ("r1", Affine8), ("c0", Affine8),
                ("c1", Affine8), ("r_step", C.c_uint32), ("c_step", C.c_uint32),
                ("p0", Affine8), ("p1", Affine8)]


class Kernel(C.Structure):
    _fields_ = [("work", Affine8), ("per_iter", C.c_uint32)]


class KX(C.Structure):
    _fields_ = [("tpb", C.c_uint32), ("ipt", C.c_uint32), ("regs", C.c_uint32),
                ("smem", C.c_uint32), ("total", C.c_double), ("coal", C.c_double),
                ("uncoal", C.c_double), ("upm", C.c_double), ("lbpw", C.c_double),
                ("synch", C.c_double)]


class Skeleton(C.Structure):
    _fields_ = [("n_kernels", C.c_uint32), ("n_arrays", C.c_uint32),
                ("n_regions", C.c_uint32), ("n_xforms", C.c_uint32),
                ("kernels", C.POINTER(Kernel)), ("arrays", C.POINTER(Array)),
                ("regions", C.POINTER(Region)), ("kx", C.POINTER(KX)), ("hull", C.c_uint32)]


class GPU(C.Structure):
    _fields_ = [("n_sm", C.c_uint32), ("warp_size", C.c_uint32), ("max_tpb", C.c_uint32),
                ("max_bps", C.c_uint32), ("max_tps", C.c_uint32), ("regs_sm", C.c_uint32),
                ("smem_sm", C.c_uint32), ("freq", C.c_double), ("mem_bw", C.c_double),
                ("mem_ld", C.c_double), ("dd_coal", C.c_double), ("dd_uncoal", C.c_double),
                ("issue", C.c_double)]


class Link(C.Structure):
    _fields_ = [("alpha", C.c_double), ("beta", C.c_double)]


class Best(C.Structure):
    _fields_ = [("t_total_s", C.c_double), ("index", C.c_uint64), ("h2d_bytes", C.c_uint64),
                ("d2h_bytes", C.c_uint64), ("n_invalid", C.c_uint64), ("n_valid", C.c_uint64)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB_PATH)
        u32p = np.ctypeslib.ndpointer(np.uint32, flags="C")
        u64p = np.ctypeslib.ndpointer(np.uint64, flags="C")
        f64p = np.ctypeslib.ndpointer(np.float64, flags="C")
        SK = C.POINTER(Skeleton)
        L.oracle_fit_pcie.argtypes = [C.c_double, C.c_double, C.c_uint64, C.POINTER(Link)]
        L.oracle_pcie_time.argtypes = [C.POINTER(Link), C.c_uint64]
        L.oracle_pcie_time.restype = C.c_double
        LP = C.POINTER(Link)
        L.oracle_choose_memory.argtypes = [LP, LP, LP, LP, LP, C.c_uint64, C.c_uint64, C.c_uint64,
                                           C.POINTER(C.c_double), C.POINTER(C.c_double),
                                           C.POINTER(C.c_int)]
        L.oracle_affine8.argtypes = [C.POINTER(Affine8), C.c_int64, C.c_int64]
        L.oracle_affine8.restype = C.c_int64
        L.oracle_usage.argtypes = [SK, C.c_int64, C.c_int64, u64p, u64p]
        L.oracle_bitmap_usage.argtypes = [SK, C.c_int64, C.c_int64, u64p, u64p]
        L.oracle_usage_hull.argtypes = [SK, C.c_int64, C.c_int64, u64p, u64p]
        L.oracle_kernel_time.argtypes = [SK, C.POINTER(GPU), C.c_uint32, C.c_uint32,
                                         C.c_int64, C.c_int64, C.POINTER(C.c_int)]
        L.oracle_kernel_time.restype = C.c_double
        L.oracle_eval_one.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.POINTER(Link),
                                      C.POINTER(Link), C.c_uint32, C.c_uint32, C.c_uint32,
                                      C.c_uint32, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64),
                                      C.POINTER(C.c_double)]
        L.oracle_eval.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.POINTER(Link),
                                  C.POINTER(Link), u32p, u32p, u32p, u32p, C.c_uint64, C.c_int,
                                  u64p, u64p, f64p]
        L.oracle_best.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.POINTER(Link),
                                  C.POINTER(Link), u32p, u32p, u32p, u32p, C.c_uint64,
                                  C.c_uint64, C.c_int, C.POINTER(Best)]
        L.oracle_eval_parts_one.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.POINTER(Link),
                                            C.POINTER(Link), C.c_uint32, C.c_uint32, C.c_uint32,
                                            C.c_uint32] + [C.POINTER(C.c_double)] * 4
        LPm = C.POINTER(Link)
        L.oracle_eval_mem_one.argtypes = [SK, C.c_uint32, C.POINTER(GPU), LPm, LPm, LPm, LPm, LPm,
                                          C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                          C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)] + \
            [C.POINTER(C.c_double)] * 3
        L.oracle_group_best.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.POINTER(Link),
                                        C.POINTER(Link), u32p, u32p, u32p, u32p, C.c_uint64,
                                        C.c_uint64, C.c_uint64, u64p, u64p, u64p, f64p]
        L.oracle_group_best.restype = C.c_uint64
        for name in ("oracle_error_magnitude", "oracle_speedup", "oracle_speedup_error"):
            getattr(L, name).argtypes = [C.c_double, C.c_double]
            getattr(L, name).restype = C.c_double
        L.oracle_crossover.argtypes = [C.c_double] * 5 + [C.POINTER(C.c_double),
                                                          C.POINTER(C.c_uint64)]
        L.oracle_op_tally_one.argtypes = [SK, C.c_uint32, C.POINTER(GPU), C.c_uint32, C.c_uint32,
                                          C.c_uint32, C.c_uint32, C.c_uint32] + \
            [C.POINTER(C.c_double)] * 3
        L.oracle_op_tally.argtypes = [SK, C.c_uint32, C.POINTER(GPU), u32p, u32p, u32p, u32p,
                                      C.c_uint64, C.c_uint32, f64p]
        L.oracle_op_tally.restype = C.c_uint64
        L.oracle_mean.argtypes = [f64p, C.c_uint64]
        L.oracle_mean.restype = C.c_double
        _lib = L
    return _lib


_MODES = {"R": 1, "W": 2, "RW": 3}


def _planes_of(skel, a):
    """The planes expression of array a (a region's default upper plane)."""
    arrs = skel["arrays"]
    return arrs[a].get("planes", (1, 0, 0, 0)) if 0 <= a < len(arrs) else (1, 0, 0, 0)


def _a8(t):
    return Affine8(*[int(v) for v in t])


class SkeletonSet:
    """Owns the ctypes arrays of one or more skeleton dicts."""

    def __init__(self, skels):
        self._keep = []
        self.arr = (Skeleton * len(skels))()
        for i, s in enumerate(skels):
            ks = (Kernel * len(s["kernels"]))(*[Kernel(_a8(k["work"]), int(k["per_iter"]))
                                               for k in s["kernels"]])
            ars = (Array * len(s["arrays"]))(*[Array(_a8(a["rows"]), _a8(a["cols"]),
                                                     a["elem_bytes"], int(a["liveout"]),
                                                     _a8(a.get("planes", (1, 0, 0, 0))))
                                               for a in s["arrays"]])
            # planes of a region: [p0, p1), default every plane of its array
            rs = (Region * max(1, len(s["regions"])))(*[
                Region(r["kernel"], r["array"], _MODES[r["mode"]], int(r["whole"]),
                       _a8(r["r0"]), _a8(r["r1"]), _a8(r["c0"]), _a8(r["c1"]),
                       int(r.get("r_step", 1)), int(r.get("c_step", 1)),
                       _a8(r.get("p0", (0, 0, 0, 0))),
                       _a8(r.get("p1", _planes_of(s, r["array"]))))
                for r in s["regions"]])
            flat = [c for row in s["kx"] for c in row]
            kx = (KX * len(flat))(*[KX(c["tpb"], c["ipt"], c["regs"], c["smem"], c["total"],
                                       c["coal"], c["uncoal"], c["upm"], c["lbpw"], c["synch"])
                                    for c in flat])
            self._keep += [ks, ars, rs, kx]
            self.arr[i] = Skeleton(len(s["kernels"]), len(s["arrays"]), len(s["regions"]),
                                   len(s["kx"]), ks, ars, rs, kx, int(bool(s.get("hull", False))))
        self.n = len(skels)

    def ptr(self, i=0):
        return C.pointer(self.arr[i])


def gpu_struct(g):
    return GPU(g["n_sm"], g["warp_size"], g["max_threads_per_block"], g["max_blocks_per_sm"],
               g["max_threads_per_sm"], g["regs_per_sm"], g["smem_per_sm"], g["freq_hz"],
               g["mem_bw_Bps"], g["mem_ld_cycles"], g["dep_del_coal"], g["dep_del_uncoal"],
               g["issue_cycles"])


def fit_pcie(t_small, t_large, large_bytes):
    out = Link()
    rc = lib().oracle_fit_pcie(t_small, t_large, large_bytes, C.byref(out))
    return rc, out


def pcie_time(link, nbytes):
    return lib().oracle_pcie_time(C.byref(link), nbytes)


def choose_memory(pin_h2d, pin_d2h, page_h2d, page_d2h, pin_alloc, h2d, d2h, footprint):
    """NEXT-4 reading 17 -> (rc, t_pinned, t_pageable, memory: 0 pinned / 1 pageable)."""
    tp, tg, m = C.c_double(), C.c_double(), C.c_int()
    rc = lib().oracle_choose_memory(*[C.byref(x) for x in (pin_h2d, pin_d2h, page_h2d, page_d2h,
                                                            pin_alloc)],
                                    h2d, d2h, footprint, C.byref(tp), C.byref(tg), C.byref(m))
    return rc, tp.value, tg.value, m.value


def affine8(coef, nx, ny):
    return lib().oracle_affine8(C.byref(_a8(coef)), nx, ny)


def usage(skel, nx, ny, bitmap=False):
    ss = SkeletonSet([skel])
    n = len(skel["arrays"])
    h = np.zeros(n, np.uint64)
    d = np.zeros(n, np.uint64)
    if bitmap:
        rc = lib().oracle_bitmap_usage(ss.ptr(), nx, ny, h, d)
        if rc != 0:
            raise ValueError("bitmap too large")
    else:
        lib().oracle_usage(ss.ptr(), nx, ny, h, d)
    return h, d


def kernel_time(skel, gpu, xform, k, nx, ny):
    ss = SkeletonSet([skel])
    reg = C.c_int(0)
    t = lib().oracle_kernel_time(ss.ptr(), C.byref(gpu_struct(gpu)), xform, k, nx, ny,
                                 C.byref(reg))
    return t, reg.value


class Problem:
    """A design space (skeleton list + GPU model + PCIe links) for batch calls."""

    def __init__(self, skels, gpu, h2d_link, d2h_link=None):
        self.ss = SkeletonSet(skels)
        self.gpu = gpu_struct(gpu)
        self.hl = h2d_link
        self.dl = d2h_link if d2h_link is not None else h2d_link

    def eval_one(self, skx, nx, ny, iters):
        h, d, t = C.c_uint64(), C.c_uint64(), C.c_double()
        ok = lib().oracle_eval_one(self.ss.arr, self.ss.n, C.byref(self.gpu), C.byref(self.hl),
                                   C.byref(self.dl), skx, nx, ny, iters, C.byref(h),
                                   C.byref(d), C.byref(t))
        return bool(ok), h.value, d.value, t.value

    def eval(self, rec, nthreads=None):
        n = len(rec["skx"])
        nthreads = nthreads or os.cpu_count() or 1
        h = np.zeros(n, np.uint64)
        d = np.zeros(n, np.uint64)
        t = np.zeros(n, np.float64)
        a = [np.ascontiguousarray(rec[k], dtype=np.uint32) for k in ("skx", "nx", "ny", "iters")]
        lib().oracle_eval(self.ss.arr, self.ss.n, C.byref(self.gpu), C.byref(self.hl),
                          C.byref(self.dl), *a, n, nthreads, h, d, t)
        return h, d, t

    def eval_mem_one(self, links, skx, nx, ny, iters):
        """links = (pin_h2d, pin_d2h, page_h2d, page_d2h, pin_alloc) as Link;
        -> (ok, h2d, d2h, t, t_h2d, t_d2h) with the per-array memory choice."""
        h, d = C.c_uint64(), C.c_uint64()
        t, th, td = C.c_double(), C.c_double(), C.c_double()
        ok = lib().oracle_eval_mem_one(self.ss.arr, self.ss.n, C.byref(self.gpu),
                                       *[C.byref(x) for x in links], skx, nx, ny, iters,
                                       C.byref(h), C.byref(d), C.byref(t), C.byref(th), C.byref(td))
        return bool(ok), h.value, d.value, t.value, th.value, td.value

    def eval_parts_one(self, skx, nx, ny, iters):
        v = [C.c_double() for _ in range(4)]
        ok = lib().oracle_eval_parts_one(self.ss.arr, self.ss.n, C.byref(self.gpu),
                                         C.byref(self.hl), C.byref(self.dl), skx, nx, ny, iters,
                                         *[C.byref(x) for x in v])
        return bool(ok), tuple(x.value for x in v)

    def group_best(self, rec, index_base=0):
        n = len(rec["skx"])
        cap = max(1, n)
        first = np.zeros(cap, np.uint64)
        count = np.zeros(cap, np.uint64)
        bi = np.zeros(cap, np.uint64)
        bt = np.zeros(cap, np.float64)
        a = [np.ascontiguousarray(rec[k], dtype=np.uint32) for k in ("skx", "nx", "ny", "iters")]
        ng = lib().oracle_group_best(self.ss.arr, self.ss.n, C.byref(self.gpu), C.byref(self.hl),
                                     C.byref(self.dl), *a, n, index_base, cap, first, count, bi, bt)
        return first[:ng], count[:ng], bi[:ng], bt[:ng]

    def op_tally_one(self, skx, nx, ny, iters, X=16):
        """(ok, fp64, int, cvt) algorithmic ops of one candidate (oracle.c)."""
        v = [C.c_double() for _ in range(3)]
        ok = lib().oracle_op_tally_one(self.ss.arr, self.ss.n, C.byref(self.gpu), skx, nx, ny,
                                       iters, X, *[C.byref(x) for x in v])
        return bool(ok), v[0].value, v[1].value, v[2].value

    def op_tally(self, rec, X=16):
        """Mean {fp64, int, cvt} ops per valid record of a batch."""
        m = np.zeros(3, np.float64)
        a = [np.ascontiguousarray(rec[k], dtype=np.uint32) for k in ("skx", "nx", "ny", "iters")]
        nv = lib().oracle_op_tally(self.ss.arr, self.ss.n, C.byref(self.gpu), *a, len(a[0]), X, m)
        return {"fp64": float(m[0]), "int": float(m[1]), "cvt": float(m[2]), "n_valid": int(nv)}

    def best(self, rec, index_base=0, nthreads=None):
        n = len(rec["skx"])
        nthreads = nthreads or os.cpu_count() or 1
        b = Best()
        a = [np.ascontiguousarray(rec[k], dtype=np.uint32) for k in ("skx", "nx", "ny", "iters")]
        rc = lib().oracle_best(self.ss.arr, self.ss.n, C.byref(self.gpu), C.byref(self.hl),
                               C.byref(self.dl), *a, n, index_base, nthreads, C.byref(b))
        return rc, b


def error_magnitude(pred, meas):
    return lib().oracle_error_magnitude(pred, meas)


def mean(v):
    v = np.ascontiguousarray(v, dtype=np.float64)
    return lib().oracle_mean(v, len(v))


def speedup(t_cpu, t_gpu):
    return lib().oracle_speedup(t_cpu, t_gpu)


def speedup_error(s_pred, s_meas):
    return lib().oracle_speedup_error(s_pred, s_meas)


def crossover(t_iter, t_once, t_h2d, t_d2h, c):
    """(n_be, iters_min): break-even iteration count (oracle.h)."""
    v, m = C.c_double(), C.c_uint64()
    lib().oracle_crossover(t_iter, t_once, t_h2d, t_d2h, c, C.byref(v), C.byref(m))
    return v.value, m.value
