"""Oracle pins: kernel-time projection (DESIGN.md §3 N5).

PAPER.md does not print the GPU model: it defers to GROPHECY [15] (P:L13, L67,
L123), built on Hong & Kim's MWP/CWP model [6].  The reading N5 is
therefore pinned only to HAND-DERIVED closed forms of that reading: every case
below is worked by hand in the docstring, with intermediates chosen to be exact
binary fractions so the expected value is exact (the final "/ freq" is a single
IEEE division of an exact integer/dyadic cycle count).  Each H&K regime, the
occupancy limits, the small-grid MWP_peak_BW term, the synchronisation cost and
the infeasible / empty special cases get one.
"""
import copy
import math

import pytest

from tests.tiny import DUMMY_KX


def kx(tpb, ipt, regs, smem, total, coal, uncoal, synch, upm=32.0, lbpw=128.0):
    return {"tpb": tpb, "ipt": ipt, "regs": regs, "smem": smem, "total": total,
            "coal": coal, "uncoal": uncoal, "upm": upm, "lbpw": lbpw, "synch": synch}


def one_kernel(work, c):
    return {"name": "k", "arrays": [], "regions": [],
            "kernels": [{"name": "k", "work": work, "per_iter": True}], "kx": [[c]]}


STENCIL_W = (4, -16, -16, 8)  # (nx-2)(ny-2)


def test_case1_fx5600(O, sk):
    """FX5600; W = 62*62 = 3844; tpb 256, naive (total 40, coal 10, regs 12).
    occ = min(8, 768/256=3, 8192/(12*256)=2) = 2; wpb = 8; ipb = 256;
    mem = 10, comp = 4*40 = 160; coal only -> ml = 420, dd = 4, mwp0 = 105,
    memc = 4200, cwpf = 4360/160 = 27.25, cpm = 16.
    blocks = ceil(3844/256) = 16; asm = 16; abps = min(2, 1) = 1; N = 8; rep = 1.
    mpk = bwr/16 ~ 11.67 -> mwp = min(105, 11.67, 8) = 8 = N; cwp = min(27.25, 8) = 8
    -> case 1: cyc = 4200 + 160 + 16*7 = 4472; no synch."""
    s = one_kernel(STENCIL_W, kx(256, 1, 12, 0, 40.0, 10.0, 0.0, 0.0))
    t, reg = O.kernel_time(s, sk.FX5600, 0, 0, 64, 64)
    assert reg == 1
    assert t == 4472 / 1.35e9


def test_case3_with_synch(O, sk):
    """tpb 64, smem variant (total 48, coal 2.25, synch 1, regs 14, smem 384).
    occ = min(8, 12, 8192/896=9, 16384/384=42) = 8; wpb = 2; ipb = 64.
    mem = 2.25, comp = 192; ml = 420, dd = 4, memc = 420*2.25 = 945,
    cwpf = 1137/192 = 5.921875.
    blocks = ceil(3844/64) = 61; asm = 16; abps = min(8, ceil(61/16)=4) = 4;
    N = 8; rep = 61/64.  mwp = min(105, ~11.67, 8) = 8; cwp = 5.921875.
    mwp == N but cwp != N; cwp < mwp and comp (192) < memc (945) -> case 3:
    cyc = (420 + 192*8) * 61/64 = 1956*61/64 = 1864.3125;
    synch = dd*(mwp-1)*1*abps*rep = 4*7*4*61/64 = 106.75; total 1971.0625."""
    s = one_kernel(STENCIL_W, kx(64, 1, 14, 384, 48.0, 2.25, 0.0, 1.0))
    t, reg = O.kernel_time(s, sk.FX5600, 0, 0, 64, 64)
    assert reg == 3
    assert t == 1971.0625 / 1.35e9


def test_case2_mwp0_binds(O, sk):
    """tpb 64, uncoalesced (total 40, uncoal 10, regs 12): occ = 8; wpb 2; ipb 64.
    mlu = 420 + 31*10 = 730; wu = 1 -> ml = 730, dd = 320, mwp0 = 730/320 = 2.28125;
    memc = 7300; cwpf = 7460/160 = 46.625; cpm = 16.
    blocks 61, abps 4, N 8, rep 61/64.  mwp = 2.28125 (mpk ~ 20.3), cwp = 8
    -> case 2: cyc = (7300*8/2.28125 + 16*1.28125) * 61/64
                 = (25600 + 20.5) * 61/64 = 24419.5390625."""
    s = one_kernel(STENCIL_W, kx(64, 1, 12, 0, 40.0, 0.0, 10.0, 0.0))
    t, reg = O.kernel_time(s, sk.FX5600, 0, 0, 64, 64)
    assert reg == 2
    assert t == 24419.5390625 / 1.35e9


# A GPU whose bandwidth terms are exact: freq 1e9, Mem_LD 512, 40 GB/s, 16 SMs
EXACT_GPU = {"n_sm": 16, "warp_size": 32, "max_threads_per_block": 512,
             "max_blocks_per_sm": 8, "max_threads_per_sm": 768, "regs_per_sm": 8192,
             "smem_per_sm": 16384, "freq_hz": 1e9, "mem_bw_Bps": 4e10,
             "mem_ld_cycles": 512.0, "dep_del_coal": 4.0, "dep_del_uncoal": 10.0,
             "issue_cycles": 4.0}


def test_case2_bandwidth_binds_full_grid(O):
    """EXACT_GPU, tpb 512 naive (regs 12): occ = min(8, 1, 8192/6144=1) = 1; wpb 16.
    coal 10: ml = 512, dd = 4, mwp0 = 128; BW_per_warp = 1e9*128/512 = 2.5e8;
    bwr = 4e10/2.5e8 = 160; memc = 5120; comp = 160; cwpf = 33; cpm = 16.
    nx = ny = 256: W = 254^2 = 64516; blocks = ceil(64516/512) = 127; asm = 16;
    abps = 1; N = 16; rep = 127/16.  mpk = 160/16 = 10 -> mwp = 10; cwp = 16
    -> case 2: cyc = (5120*16/10 + 16*9) * 127/16 = 8336*127/16 = 66167."""
    s = one_kernel(STENCIL_W, kx(512, 1, 12, 0, 40.0, 10.0, 0.0, 0.0))
    t, reg = O.kernel_time(s, EXACT_GPU, 0, 0, 256, 256)
    assert reg == 2
    assert t == 66167 / 1e9


def test_small_grid_uses_active_sms(O):
    """Same kernel at 64x64: blocks = ceil(3844/512) = 8 < 16 SMs, so
    #Active_SMs = 8 and MWP_peak_BW = 160/8 = 20 (not 160/16 = 10):
    mwp = min(128, 20, 16) = 16 = N, cwp = 16 = N -> case 1 with rep = 1:
    cyc = 5120 + 160 + 16*15 = 5520."""
    s = one_kernel(STENCIL_W, kx(512, 1, 12, 0, 40.0, 10.0, 0.0, 0.0))
    t, reg = O.kernel_time(s, EXACT_GPU, 0, 0, 64, 64)
    assert reg == 1
    assert t == 5520 / 1e9


def test_no_memory_instructions(O, sk):
    """coal = uncoal = 0: pure issue time, cyc = Comp_cycles * N * #Rep.
    tpb 128, total 40, no regs/smem limit: occ = min(8, 6) = 6; wpb 4;
    blocks = ceil(3844/128) = 31; asm 16; abps = min(6, 2) = 2; N = 8;
    rep = 31/32; cyc = 160*8*31/32 = 1240."""
    s = one_kernel(STENCIL_W, kx(128, 1, 0, 0, 40.0, 0.0, 0.0, 2.0))
    t, reg = O.kernel_time(s, sk.FX5600, 0, 0, 64, 64)
    assert reg == 4
    assert t == 1240 / 1.35e9


@pytest.mark.parametrize("c", [kx(1024, 1, 0, 0, 40.0, 10.0, 0.0, 0.0),   # tpb > 512
                               kx(512, 2, 20, 0, 70.0, 17.0, 0.0, 0.0),   # 20*512 regs > 8192
                               kx(64, 1, 0, 20000, 40.0, 10.0, 0.0, 0.0)])  # smem > 16 KiB
def test_infeasible_is_infinite(O, sk, c):
    t, reg = O.kernel_time(one_kernel(STENCIL_W, c), sk.FX5600, 0, 0, 64, 64)
    assert reg == -1 and math.isinf(t) and t > 0


def test_no_work_is_zero(O, sk):
    # (nx-2)(ny-2) = 0 at 2x2; negative work clamps to 0
    c = kx(256, 1, 12, 0, 40.0, 10.0, 0.0, 0.0)
    t, reg = O.kernel_time(one_kernel(STENCIL_W, c), sk.FX5600, 0, 0, 2, 2)
    assert reg == 0 and t == 0.0
    t, reg = O.kernel_time(one_kernel((-5, 0, 0, 0), c), sk.FX5600, 0, 0, 100, 100)
    assert reg == 0 and t == 0.0


def test_occupancy_limits_change_rep(O, sk):
    """Raising registers so occupancy drops from 2 to 1 doubles #Rep at a
    saturated grid: tpb 256, naive, 8192x8192 grid with W = nx*ny:
    blocks = 2^26/256 = 262144; occ 2 -> rep = 262144/32 = 8192; occ 1 (regs 20
    -> 8192/5120 = 1) -> N halves too.  Both are pure case-1/2 forms; check the
    ratio of #Rep via the no-memory variant: cyc = 160 * N * rep."""
    c2 = kx(256, 1, 12, 0, 40.0, 0.0, 0.0, 0.0)   # occ 2: N = 16, rep = 8192
    c1 = kx(256, 1, 20, 0, 40.0, 0.0, 0.0, 0.0)   # occ 1: N = 8,  rep = 16384
    t2, _ = O.kernel_time(one_kernel((0, 0, 0, 8), c2), sk.FX5600, 0, 0, 8192, 8192)
    t1, _ = O.kernel_time(one_kernel((0, 0, 0, 8), c1), sk.FX5600, 0, 0, 8192, 8192)
    assert t2 == 160 * 16 * 8192 / 1.35e9
    assert t1 == 160 * 8 * 16384 / 1.35e9


def test_skeleton_xform_indexing(O, sk):
    """kx is [xform][kernel]: a 2-kernel skeleton with distinct per-kernel
    entries must pick entry (x, k)."""
    c_fast = kx(128, 1, 0, 0, 40.0, 0.0, 0.0, 0.0)
    c_slow = kx(128, 1, 0, 0, 80.0, 0.0, 0.0, 0.0)
    s = {"name": "two", "arrays": [], "regions": [],
         "kernels": [{"name": "a", "work": STENCIL_W, "per_iter": True}] * 2,
         "kx": [[c_fast, c_slow], [c_slow, c_fast]]}
    t00, _ = O.kernel_time(s, sk.FX5600, 0, 0, 64, 64)
    t01, _ = O.kernel_time(s, sk.FX5600, 0, 1, 64, 64)
    t10, _ = O.kernel_time(s, sk.FX5600, 1, 0, 64, 64)
    assert t00 == 1240 / 1.35e9 and t01 == 2480 / 1.35e9 and t10 == t01
