"""Thin Python binding of libgrophecy.so (include/grophecy.h).

Argument marshalling only: every step of the projection runs in the CUDA
library.  PyTorch supplies device memory (tensors) and streams.  There is no
fallback: if the shared library is missing or fails to load, importing this
module raises.
"""
import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# GROPHECY_LIB: an alternative in-tree build of the same library (A/B
# measurements of build variants, scripts/ab_lib.sh)
LIB_PATH = os.environ.get("GROPHECY_LIB") or os.path.join(HERE, "libgrophecy.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} not built; run `python -m paper_conf_ipps_boyermk13_b200.build` "
        "(there is no CPU fallback)")
_L = C.CDLL(LIB_PATH)

OK, EINVAL, ELIMIT, ECUDA, ENOFEASIBLE, EBADCAND = 0, -1, -2, -3, -5, -6
ARRAY_LIVEOUT = 1
R, W = 1, 2
REGION_WHOLE = 1
SKEL_HULL = 1
KERNEL_PER_ITER = 1
DIR_H2D, DIR_D2H = 0, 1
UINT64_MAX = 2**64 - 1


class GrophecyError(RuntimeError):
    def __init__(self, code, where):
        self.code = code
        msg = _L.grophecy_last_error().decode(errors="replace")
        super().__init__(f"{where}: status {code}: {msg}")


class Link(C.Structure):
    _fields_ = [("alpha_s", C.c_double), ("beta_s_per_byte", C.c_double)]


class PCIe(C.Structure):
    _fields_ = [("h2d", Link), ("d2h", Link)]


class MemoryModel(C.Structure):
    """grophecy_memory_model (NEXT-4): pinned / pageable links + pinned allocation."""
    _fields_ = [("pinned", PCIe), ("pageable", PCIe), ("pin_alloc", Link)]


class MemoryChoice(C.Structure):
    _fields_ = [("t_pinned_s", C.c_double), ("t_pageable_s", C.c_double),
                ("memory", C.c_int32), ("reserved", C.c_int32)]


class Affine8(C.Structure):
    _fields_ = [("c0", C.c_int32), ("c1", C.c_int32), ("c2", C.c_int32), ("c3", C.c_int32)]


class ArrayDesc(C.Structure):
    _fields_ = [("rows", Affine8), ("cols", Affine8), ("elem_bytes", C.c_uint32),
                ("flags", C.c_uint32), ("planes", Affine8)]


class RegionDesc(C.Structure):
    _fields_ = [("kernel", C.c_uint8), ("array", C.c_uint8), ("mode", C.c_uint8),
                ("flags", C.c_uint8), ("r0", Affine8), ("r1", Affine8), ("c0", Affine8),
                ("c1", Affine8), ("r_step", C.c_uint16), ("c_step", C.c_uint16),
                ("p0", Affine8), ("p1", Affine8)]


class KernelDesc(C.Structure):
    _fields_ = [("work_items", Affine8), ("flags", C.c_uint32)]


class KxDesc(C.Structure):
    _fields_ = [("tpb", C.c_uint32), ("ipt", C.c_uint32), ("regs_per_thread", C.c_uint32),
                ("smem_per_block", C.c_uint32), ("total_insts", C.c_double),
                ("coal_insts", C.c_double), ("uncoal_insts", C.c_double),
                ("uncoal_per_mw", C.c_double), ("load_bytes_per_warp", C.c_double),
                ("synch_insts", C.c_double)]


class SkeletonDesc(C.Structure):
    _fields_ = [("n_kernels", C.c_uint32), ("n_arrays", C.c_uint32), ("n_regions", C.c_uint32),
                ("n_xforms", C.c_uint32), ("kernels", C.POINTER(KernelDesc)),
                ("arrays", C.POINTER(ArrayDesc)), ("regions", C.POINTER(RegionDesc)),
                ("kx", C.POINTER(KxDesc)), ("flags", C.c_uint32), ("reserved", C.c_uint32)]


class GpuModel(C.Structure):
    _fields_ = [("n_sm", C.c_uint32), ("warp_size", C.c_uint32),
                ("max_threads_per_block", C.c_uint32), ("max_blocks_per_sm", C.c_uint32),
                ("max_threads_per_sm", C.c_uint32), ("regs_per_sm", C.c_uint32),
                ("smem_per_sm", C.c_uint32), ("freq_hz", C.c_double), ("mem_bw_Bps", C.c_double),
                ("mem_ld_cycles", C.c_double), ("dep_del_coal", C.c_double),
                ("dep_del_uncoal", C.c_double), ("issue_cycles", C.c_double)]


class Batch(C.Structure):
    _fields_ = [("skx", C.c_void_p), ("nx", C.c_void_p), ("ny", C.c_void_p),
                ("iters", C.c_void_p), ("n", C.c_uint64), ("index_base", C.c_uint64),
                ("stripe_len", C.c_uint64), ("stripe_stride", C.c_uint64)]


class BestResult(C.Structure):
    _fields_ = [("t_total_s", C.c_double), ("index", C.c_uint64), ("h2d_bytes", C.c_uint64),
                ("d2h_bytes", C.c_uint64), ("n_invalid", C.c_uint64), ("n_valid", C.c_uint64)]

    def as_tuple(self):
        return (self.t_total_s, self.index, self.h2d_bytes, self.d2h_bytes, self.n_invalid,
                self.n_valid)


assert C.sizeof(BestResult) == 48 and C.sizeof(RegionDesc) == 104 and C.sizeof(ArrayDesc) == 56 and C.sizeof(KxDesc) == 64
assert C.sizeof(SkeletonDesc) == 56


class Parts(C.Structure):
    _fields_ = [("t_iter_s", C.c_void_p), ("t_once_s", C.c_void_p), ("t_h2d_s", C.c_void_p),
                ("t_d2h_s", C.c_void_p)]


class GroupResult(C.Structure):
    _fields_ = [("best_t_s", C.c_double), ("first", C.c_uint64), ("count", C.c_uint64),
                ("best_index", C.c_uint64), ("h2d_bytes", C.c_uint64), ("d2h_bytes", C.c_uint64)]


class SynthRule(C.Structure):
    _fields_ = [("kind", C.c_uint32), ("lo", C.c_uint32), ("hi", C.c_uint32),
                ("it_lo", C.c_uint32), ("it_hi", C.c_uint32), ("pad", C.c_uint32)]


_vp = C.c_void_p
_sig = {
    "grophecy_fit_pcie": (C.c_int, [C.c_double, C.c_double, C.c_uint64, C.POINTER(Link)]),
    "grophecy_pcie_time": (C.c_double, [C.POINTER(Link), C.c_uint64]),
    "grophecy_space_validate": (C.c_int, [C.POINTER(SkeletonDesc), C.c_uint32, C.POINTER(GpuModel)]),
    "grophecy_space_create": (C.c_int, [C.POINTER(SkeletonDesc), C.c_uint32, C.POINTER(GpuModel),
                                        C.c_int, C.POINTER(_vp)]),
    "grophecy_space_destroy": (None, [_vp]),
    "grophecy_eval": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), _vp, _vp, _vp, _vp]),
    "grophecy_invalid_count": (C.c_int, [_vp, C.POINTER(C.c_uint64), _vp]),
    "grophecy_best_allreduce": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), _vp,
                                          C.POINTER(BestResult), _vp]),
    "grophecy_nccl_unique_id": (C.c_int, [_vp]),
    "grophecy_nccl_comm_init": (C.c_int, [C.c_int, C.c_int, _vp, C.c_int, C.POINTER(_vp)]),
    "grophecy_nccl_comm_destroy": (C.c_int, [_vp]),
    "grophecy_eval_mem": (C.c_int, [_vp, C.POINTER(MemoryModel), C.POINTER(Batch), _vp, _vp, _vp,
                                    _vp, _vp]),
    "grophecy_best_mem": (C.c_int, [_vp, C.POINTER(MemoryModel), C.POINTER(Batch),
                                    C.POINTER(BestResult), _vp]),
    "grophecy_eval_parts": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), _vp, _vp, _vp,
                                      C.POINTER(Parts), _vp]),
    "grophecy_group_best": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), _vp, C.c_uint64,
                                      C.POINTER(C.c_uint64), _vp]),
    "grophecy_group_merge_host": (C.c_int, [C.POINTER(GroupResult), C.POINTER(GroupResult),
                                            C.POINTER(GroupResult)]),
    "grophecy_group_speedup": (C.c_int, [_vp, _vp, C.c_uint64, _vp, _vp]),
    "grophecy_crossover": (C.c_int, [_vp, _vp, _vp, _vp, _vp, C.c_double, C.c_uint64, _vp, _vp,
                                     _vp]),
    "grophecy_speedup": (C.c_double, [C.c_double, C.c_double]),
    "grophecy_error_magnitude": (C.c_double, [C.c_double, C.c_double]),
    "grophecy_mean": (C.c_double, [C.POINTER(C.c_double), C.c_uint64]),
    "grophecy_best": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), C.POINTER(BestResult), _vp]),
    "grophecy_best_async": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), _vp, C.c_int, _vp]),
    "grophecy_best_combine": (C.c_int, [_vp, C.c_uint32, _vp, _vp]),
    "grophecy_best_combine_host": (C.c_int, [C.POINTER(BestResult), C.c_uint32, C.POINTER(BestResult)]),
    "grophecy_best_host": (C.c_int, [_vp, C.POINTER(PCIe), C.POINTER(Batch), C.POINTER(BestResult),
                                     _vp]),
    "grophecy_best_allreduce_result": (C.c_int, [_vp, _vp, _vp, C.POINTER(BestResult), _vp]),
    "grophecy_measure_transfer": (C.c_int, [C.c_int, C.c_int, C.c_uint64, C.c_int, C.c_int,
                                            C.POINTER(C.c_double), C.POINTER(C.c_double)]),
    "grophecy_calibrate": (C.c_int, [C.c_int, C.c_int, C.c_uint64, C.POINTER(PCIe)]),
    "grophecy_measure_transfer_mem": (C.c_int, [C.c_int, C.c_int, C.c_int, C.c_uint64, C.c_int,
                                                C.c_int, C.POINTER(C.c_double),
                                                C.POINTER(C.c_double)]),
    "grophecy_measure_pin_alloc": (C.c_int, [C.c_int, C.c_uint64, C.c_int, C.POINTER(C.c_double),
                                             C.POINTER(C.c_double)]),
    "grophecy_calibrate_memory": (C.c_int, [C.c_int, C.c_int, C.c_uint64, C.POINTER(MemoryModel)]),
    "grophecy_choose_memory": (C.c_int, [C.POINTER(MemoryModel), C.c_uint64, C.c_uint64,
                                         C.c_uint64, C.POINTER(MemoryChoice)]),
    "grophecy_synth_records": (C.c_int, [C.POINTER(SynthRule), C.c_uint32, C.c_uint64, C.c_uint32,
                                         C.c_uint64, C.c_uint64, C.c_uint64, _vp, _vp, _vp, _vp,
                                         _vp]),
    "grophecy_plan_usage_host": (C.c_int, [C.POINTER(SkeletonDesc), C.c_int64, C.c_int64,
                                           C.POINTER(C.c_uint64), C.POINTER(C.c_uint64),
                                           C.POINTER(C.c_uint32), C.POINTER(C.c_uint32)]),
    "grophecy_plan_stats": (C.c_int, [C.POINTER(SkeletonDesc), C.POINTER(C.c_uint32)]),
    "grophecy_launch_count": (C.c_uint64, []),
    "grophecy_debug_phase_cycles": (C.c_int, [C.POINTER(C.c_uint64)]),
    "grophecy_last_error": (C.c_char_p, []),
    "grophecy_abi_version": (C.c_int, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_L, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_sig)

# the struct layouts above are ABI version 4 (include/grophecy.h)
ABI_VERSION = 4
if _L.grophecy_abi_version() != ABI_VERSION:
    raise ImportError(f"libgrophecy.so ABI {_L.grophecy_abi_version()} != binding ABI {ABI_VERSION}: rebuild")


def lib():
    return _L


def _check(rc, where, ok=(OK,)):
    if rc not in ok:
        raise GrophecyError(rc, where)
    return rc


# ---------------------------------------------------------------- PCIe model
def fit_pcie(t_small_s, t_large_s, large_bytes):
    out = Link()
    _check(_L.grophecy_fit_pcie(t_small_s, t_large_s, large_bytes, C.byref(out)), "fit_pcie")
    return out


def pcie_time(link, nbytes):
    return _L.grophecy_pcie_time(C.byref(link), nbytes)


def pcie(h2d, d2h=None):
    return PCIe(h2d, d2h if d2h is not None else h2d)


# ---------------------------------------------------------------- descriptors
_MODES = {"R": R, "W": W, "RW": R | W}


def _planes_of(skel, a):
    """The planes expression of array a (a region's default upper plane)."""
    arrs = skel["arrays"]
    return arrs[a].get("planes", (1, 0, 0, 0)) if 0 <= a < len(arrs) else (1, 0, 0, 0)


def _a8(t):
    return Affine8(*[int(v) for v in t])


class Skeletons:
    """Marshals skeleton dicts (synth/skeletons.py format) into grophecy
    descriptors and keeps the ctypes buffers alive."""

    def __init__(self, skels):
        self.keep = []
        self.arr = (SkeletonDesc * len(skels))()
        for i, s in enumerate(skels):
            ks = (KernelDesc * len(s["kernels"]))(*[
                KernelDesc(_a8(k["work"]), KERNEL_PER_ITER if k["per_iter"] else 0)
                for k in s["kernels"]])
            ars = (ArrayDesc * max(1, len(s["arrays"])))(*[
                ArrayDesc(_a8(a["rows"]), _a8(a["cols"]), a["elem_bytes"],
                          ARRAY_LIVEOUT if a["liveout"] else 0,
                          _a8(a.get("planes", (1, 0, 0, 0)))) for a in s["arrays"]])
            # planes of a region: [p0, p1), default every plane of its array
            rs = (RegionDesc * max(1, len(s["regions"])))(*[
                RegionDesc(r["kernel"], r["array"], _MODES[r["mode"]],
                           REGION_WHOLE if r["whole"] else 0, _a8(r["r0"]), _a8(r["r1"]),
                           _a8(r["c0"]), _a8(r["c1"]), int(r.get("r_step", 1)),
                           int(r.get("c_step", 1)), _a8(r.get("p0", (0, 0, 0, 0))),
                           _a8(r.get("p1", _planes_of(s, r["array"]))))
                for r in s["regions"]])
            flat = [c for row in s["kx"] for c in row]
            kx = (KxDesc * len(flat))(*[
                KxDesc(c["tpb"], c["ipt"], c["regs"], c["smem"], c["total"], c["coal"],
                       c["uncoal"], c["upm"], c["lbpw"], c["synch"]) for c in flat])
            self.keep += [ks, ars, rs, kx]
            self.arr[i] = SkeletonDesc(len(s["kernels"]), len(s["arrays"]), len(s["regions"]),
                                       len(s["kx"]), ks, ars, rs, kx,
                                       SKEL_HULL if s.get("hull", False) else 0, 0)
        self.n = len(skels)


def gpu_model(g):
    return GpuModel(g["n_sm"], g["warp_size"], g["max_threads_per_block"],
                    g["max_blocks_per_sm"], g["max_threads_per_sm"], g["regs_per_sm"],
                    g["smem_per_sm"], g["freq_hz"], g["mem_bw_Bps"], g["mem_ld_cycles"],
                    g["dep_del_coal"], g["dep_del_uncoal"], g["issue_cycles"])


def validate(skels, gpu):
    sd = Skeletons(skels)
    return _L.grophecy_space_validate(sd.arr, sd.n, C.byref(gpu_model(gpu)))


# ---------------------------------------------------------------- torch glue
def _torch():
    import torch
    return torch


def _stream_ptr(stream):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


def _ptr(t):
    return C.c_void_p(t.data_ptr()) if t is not None else C.c_void_p(0)


class Records:
    """SoA candidate records in device memory (four uint32 tensors stored as
    int32; the library reads them as uint32)."""

    def __init__(self, skx, nx, ny, iters):
        self.skx, self.nx, self.ny, self.iters = skx, nx, ny, iters
        self.n = skx.numel()

    @classmethod
    def from_numpy(cls, rec, device="cuda"):
        torch = _torch()
        ts = [torch.from_numpy(np.ascontiguousarray(rec[k]).view(np.int32)).to(device)
              for k in ("skx", "nx", "ny", "iters")]
        return cls(*ts)

    @classmethod
    def empty(cls, n, device="cuda"):
        torch = _torch()
        return cls(*[torch.empty(max(n, 1), dtype=torch.int32, device=device)[:n]
                     for _ in range(4)])

    def batch(self, index_base=0, start=0, stop=None, stripe_len=0, stripe_stride=0):
        """Records [start, stop) as a grophecy_batch; with stripe_len the
        batch-local record i has global index index_base + (i // stripe_len)
        * stripe_stride + i % stripe_len (include/grophecy.h)."""
        stop = self.n if stop is None else stop
        off = start * 4
        return Batch(self.skx.data_ptr() + off, self.nx.data_ptr() + off,
                     self.ny.data_ptr() + off, self.iters.data_ptr() + off, stop - start,
                     index_base, stripe_len, stripe_stride)


def synth_rules(cfg):
    rules = (SynthRule * len(cfg["rules"]))(*[
        SynthRule(r["kind"], r["lo"], r["hi"], r["it_lo"], r["it_hi"], 0) for r in cfg["rules"]])
    return rules


def synth_records(cfg, start=0, count=None, device="cuda", stream=None, out=None):
    """Generate records [start, start+count) of config ``cfg`` on the GPU."""
    count = cfg["n"] - start if count is None else count
    rec = out if out is not None else Records.empty(count, device)
    rules = synth_rules(cfg)
    _check(_L.grophecy_synth_records(rules, len(cfg["rules"]), cfg["n"], cfg["n_xforms"],
                                     cfg["seed"], start, count, _ptr(rec.skx), _ptr(rec.nx),
                                     _ptr(rec.ny), _ptr(rec.iters), _stream_ptr(stream)),
           "synth_records")
    return rec


class Space:
    """A design space on one device (grophecy_space_create / _destroy)."""

    def __init__(self, skels, gpu, device=None):
        torch = _torch()
        self.device = torch.cuda.current_device() if device is None else device
        sd = Skeletons(skels)
        h = C.c_void_p()
        _check(_L.grophecy_space_create(sd.arr, sd.n, C.byref(gpu_model(gpu)), self.device,
                                        C.byref(h)), "space_create")
        self.h = h
        self.n_skels = sd.n

    def close(self):
        if self.h:
            _L.grophecy_space_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def eval(self, pc, rec, index_base=0, out=None, stream=None):
        torch = _torch()
        n = rec.n
        if out is None:
            dev = rec.skx.device
            out = (torch.empty(n, dtype=torch.int64, device=dev),
                   torch.empty(n, dtype=torch.int64, device=dev),
                   torch.empty(n, dtype=torch.float64, device=dev))
        b = rec.batch(index_base)
        _check(_L.grophecy_eval(self.h, C.byref(pc), C.byref(b), _ptr(out[0]), _ptr(out[1]),
                                _ptr(out[2]), _stream_ptr(stream)), "eval")
        return out

    def eval_parts(self, pc, rec, index_base=0, stream=None):
        """(h2d, d2h, t, t_iter, t_once, t_h2d, t_d2h) device tensors."""
        torch = _torch()
        n, dev = rec.n, rec.skx.device
        h = torch.empty(n, dtype=torch.int64, device=dev)
        d = torch.empty(n, dtype=torch.int64, device=dev)
        ts = [torch.empty(n, dtype=torch.float64, device=dev) for _ in range(5)]
        parts = Parts(*[t.data_ptr() for t in ts[1:]])
        b = rec.batch(index_base)
        _check(_L.grophecy_eval_parts(self.h, C.byref(pc), C.byref(b), _ptr(h), _ptr(d),
                                      _ptr(ts[0]), C.byref(parts), _stream_ptr(stream)),
               "eval_parts")
        return (h, d, *ts)

    def eval_mem(self, model, rec, index_base=0, stream=None):
        """NEXT-4: (h2d, d2h, t, t_iter, t_once, t_h2d, t_d2h) with the per-array
        pinned / pageable choice of `model` (MemoryModel)."""
        torch = _torch()
        n, dev = rec.n, rec.skx.device
        h = torch.empty(n, dtype=torch.int64, device=dev)
        d = torch.empty(n, dtype=torch.int64, device=dev)
        ts = [torch.empty(n, dtype=torch.float64, device=dev) for _ in range(5)]
        parts = Parts(*[t.data_ptr() for t in ts[1:]])
        b = rec.batch(index_base)
        _check(_L.grophecy_eval_mem(self.h, C.byref(model), C.byref(b), _ptr(h), _ptr(d),
                                    _ptr(ts[0]), C.byref(parts), _stream_ptr(stream)), "eval_mem")
        return (h, d, *ts)

    def best_allreduce(self, pc, rec, comm, index_base=0, stream=None, batch=None):
        """Global best over the ranks of NCCL communicator `comm` (NcclComm):
        this rank's shard `rec` with global index_base."""
        r = BestResult()
        b = batch if batch is not None else rec.batch(index_base)
        rc = _L.grophecy_best_allreduce(self.h, C.byref(pc), C.byref(b), comm.handle, C.byref(r),
                                        _stream_ptr(stream))
        _check(rc, "best_allreduce", ok=(OK, ENOFEASIBLE, EBADCAND))
        return rc, r

    def best_mem(self, model, rec, index_base=0, stream=None):
        r = BestResult()
        b = rec.batch(index_base)
        rc = _L.grophecy_best_mem(self.h, C.byref(model), C.byref(b), C.byref(r),
                                  _stream_ptr(stream))
        _check(rc, "best_mem", ok=(OK, ENOFEASIBLE, EBADCAND))
        return rc, r

    def group_best(self, pc, rec, index_base=0, capacity=None, stream=None, out=None,
                   as_tensor=False):
        """Best transformation per projection point: (rc, n_groups, results)
        with results a list of GroupResult, or the raw device tensor (6 int64
        per group) when as_tensor=True."""
        torch = _torch()
        cap = rec.n if capacity is None else capacity
        if out is None:
            out = torch.empty(max(1, cap) * 6, dtype=torch.int64, device=rec.skx.device)
        ng = C.c_uint64()
        b = rec.batch(index_base)
        rc = _L.grophecy_group_best(self.h, C.byref(pc), C.byref(b), _ptr(out), cap,
                                    C.byref(ng), _stream_ptr(stream))
        _check(rc, "group_best", ok=(OK, ELIMIT))
        if as_tensor:
            return rc, ng.value, out
        raw = out.cpu().numpy().tobytes()
        k = min(ng.value, cap)
        return rc, ng.value, [GroupResult.from_buffer_copy(raw[48 * i:48 * (i + 1)]) for i in range(k)]

    def invalid_count(self, stream=None):
        v = C.c_uint64()
        _check(_L.grophecy_invalid_count(self.h, C.byref(v), _stream_ptr(stream)), "invalid_count")
        return v.value

    def best(self, pc, rec, index_base=0, stream=None, batch=None):
        r = BestResult()
        b = batch if batch is not None else rec.batch(index_base)
        rc = _L.grophecy_best(self.h, C.byref(pc), C.byref(b), C.byref(r), _stream_ptr(stream))
        _check(rc, "best", ok=(OK, ENOFEASIBLE, EBADCAND))
        return rc, r

    def best_async(self, pc, batch, dout, accumulate=False, stream=None):
        _check(_L.grophecy_best_async(self.h, C.byref(pc), C.byref(batch), _ptr(dout),
                                      int(bool(accumulate)), _stream_ptr(stream)), "best_async")

    def best_host(self, pc, rec_host, index_base=0, stream=None, stripe_len=0, stripe_stride=0):
        """rec_host: dict of four uint32 arrays (numpy or pinned torch CPU tensors)."""
        ptrs = []
        for k in ("skx", "nx", "ny", "iters"):
            a = rec_host[k]
            ptrs.append(a.data_ptr() if hasattr(a, "data_ptr") else a.ctypes.data)
        n = len(rec_host["skx"])
        hb = Batch(*ptrs, n, index_base, stripe_len, stripe_stride)
        r = BestResult()
        rc = _L.grophecy_best_host(self.h, C.byref(pc), C.byref(hb), C.byref(r), _stream_ptr(stream))
        _check(rc, "best_host", ok=(OK, ENOFEASIBLE, EBADCAND))
        return rc, r

    def allreduce_result(self, dres, comm, stream=None):
        """Global best over the ranks of `comm` of a device result tensor
        (grophecy_best_allreduce_result)."""
        r = BestResult()
        rc = _L.grophecy_best_allreduce_result(self.h, _ptr(dres), comm.handle, C.byref(r),
                                               _stream_ptr(stream))
        _check(rc, "best_allreduce_result", ok=(OK, ENOFEASIBLE, EBADCAND))
        return rc, r


def nccl_unique_id():
    """128-byte ncclUniqueId (rank 0 creates, all ranks receive it)."""
    buf = (C.c_char * 128)()
    _check(_L.grophecy_nccl_unique_id(buf), "nccl_unique_id")
    return bytes(buf)


class NcclComm:
    """An ncclComm_t for grophecy_best_allreduce (one rank per GPU)."""

    def __init__(self, nranks, rank, uid, device=0):
        self.handle = C.c_void_p()
        buf = (C.c_char * 128).from_buffer_copy(uid)
        _check(_L.grophecy_nccl_comm_init(nranks, rank, buf, device, C.byref(self.handle)),
               "nccl_comm_init")

    def close(self):
        if self.handle:
            _L.grophecy_nccl_comm_destroy(self.handle)
            self.handle = C.c_void_p()


def best_result_tensor(n=1, device="cuda"):
    """A device buffer for n grophecy_best_result (48 bytes each, as int64)."""
    torch = _torch()
    return torch.empty(6 * n, dtype=torch.int64, device=device)


def best_combine(din, count, dout, stream=None):
    _check(_L.grophecy_best_combine(_ptr(din), count, _ptr(dout), _stream_ptr(stream)),
           "best_combine")


def best_combine_host(results):
    arr = (BestResult * max(1, len(results)))(*results)
    out = BestResult()
    _check(_L.grophecy_best_combine_host(arr, len(results), C.byref(out)), "best_combine_host")
    return out


def result_from_tensor(t, i=0):
    """Decode result i of a device/host tensor of 48-byte results."""
    raw = t.detach().cpu().contiguous().numpy().tobytes()
    return BestResult.from_buffer_copy(raw[48 * i:48 * (i + 1)])


def measure_transfer(device, direction, nbytes, reps=10, warmup=2):
    wall, ev = C.c_double(), C.c_double()
    _check(_L.grophecy_measure_transfer(device, direction, nbytes, reps, warmup, C.byref(wall),
                                        C.byref(ev)), "measure_transfer")
    return wall.value, ev.value


def calibrate(device=0, reps=10, large_bytes=1 << 29):
    out = PCIe()
    _check(_L.grophecy_calibrate(device, reps, large_bytes, C.byref(out)), "calibrate")
    return out


MEM_PINNED, MEM_PAGEABLE = 0, 1


def measure_transfer_mem(device, direction, memory, nbytes, reps=10, warmup=2):
    wall, ev = C.c_double(), C.c_double()
    _check(_L.grophecy_measure_transfer_mem(device, direction, memory, nbytes, reps, warmup,
                                            C.byref(wall), C.byref(ev)), "measure_transfer_mem")
    return wall.value, ev.value


def measure_pin_alloc(device, nbytes, reps=10):
    a, f = C.c_double(), C.c_double()
    _check(_L.grophecy_measure_pin_alloc(device, nbytes, reps, C.byref(a), C.byref(f)),
           "measure_pin_alloc")
    return a.value, f.value


def calibrate_memory(device=0, reps=10, large_bytes=1 << 29):
    out = MemoryModel()
    _check(_L.grophecy_calibrate_memory(device, reps, large_bytes, C.byref(out)),
           "calibrate_memory")
    return out


def choose_memory(model, h2d_bytes, d2h_bytes, footprint_bytes):
    out = MemoryChoice()
    _check(_L.grophecy_choose_memory(C.byref(model), h2d_bytes, d2h_bytes, footprint_bytes,
                                     C.byref(out)), "choose_memory")
    return out


def plan_usage_host(skel, nx, ny):
    """Host evaluation of the compiled usage plan: (rc, h2d[], d2h[], tx, ty)."""
    sd = Skeletons([skel])
    na = max(1, len(skel["arrays"]))
    h = (C.c_uint64 * na)()
    d = (C.c_uint64 * na)()
    tx, ty = C.c_uint32(), C.c_uint32()
    rc = _L.grophecy_plan_usage_host(sd.arr, nx, ny, h, d, C.byref(tx), C.byref(ty))
    n = len(skel["arrays"])
    return rc, list(h)[:n], list(d)[:n], tx.value, ty.value


def plan_stats(skel):
    sd = Skeletons([skel])
    st = (C.c_uint32 * 9)()
    rc = _L.grophecy_plan_stats(sd.arr, st)
    return rc, list(st)


def group_merge_host(a, b):
    """The group split across two consecutive batches, merged (a precedes b)."""
    out = GroupResult()
    _check(_L.grophecy_group_merge_host(C.byref(a), C.byref(b), C.byref(out)), "group_merge_host")
    return out


def group_speedup(groups, t_cpu, stream=None):
    """Predicted speedup per group: groups = the int64 device tensor
    of grophecy_group_best (6 words per group), t_cpu = float64 device tensor
    (one CPU time per group).  Returns a float64 device tensor."""
    torch = _torch()
    n = t_cpu.numel()
    out = torch.empty(n, dtype=torch.float64, device=t_cpu.device)
    _check(_L.grophecy_group_speedup(_ptr(groups), _ptr(t_cpu), n, _ptr(out), _stream_ptr(stream)),
           "group_speedup")
    return out


def crossover(t_iter, t_once, t_h2d, t_d2h, t_cpu_iter, stream=None):
    """Break-even iteration counts (n_be float64, iters_min int64 holding
    uint64 bits) from grophecy_eval_parts outputs; t_cpu_iter is a float64
    device tensor (per candidate) or a Python float (every candidate)."""
    torch = _torch()
    n = t_iter.numel()
    nbe = torch.empty(n, dtype=torch.float64, device=t_iter.device)
    imin = torch.empty(n, dtype=torch.int64, device=t_iter.device)
    vec = not isinstance(t_cpu_iter, (int, float))
    _check(_L.grophecy_crossover(_ptr(t_iter), _ptr(t_once), _ptr(t_h2d), _ptr(t_d2h),
                                 _ptr(t_cpu_iter) if vec else None,
                                 0.0 if vec else float(t_cpu_iter), n, _ptr(nbe), _ptr(imin),
                                 _stream_ptr(stream)), "crossover")
    return nbe, imin


def speedup(t_cpu, t_gpu):
    return _L.grophecy_speedup(t_cpu, t_gpu)


def mean(values):
    """grophecy_mean: arithmetic mean summed in order."""
    v = list(values)
    arr = (C.c_double * max(1, len(v)))(*v)
    return _L.grophecy_mean(arr, len(v))


def error_magnitude(pred, meas):
    return _L.grophecy_error_magnitude(pred, meas)


def launch_count():
    return _L.grophecy_launch_count()
