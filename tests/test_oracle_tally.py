"""Pins of the oracle's algorithmic op tally (oracle.c oracle_op_tally_one,
DESIGN.md §6): hand counts of its stated amortisation rule on the App. B
workloads.  The tally is a measurement convention for the op-bound roofline
(SURVEY.md §8(d)), not a quantity the paper prints.

Rule recap: per (candidate, kernel) on a saturated grid 2 int (ceil
division) + 1 conversion + fp64 {rep: 2 unless D is a power of two; E rep:
1; S rep + add: 2 unless S = 0; / freq: 2; running sum: 1}; below saturation
2 int + 1 fp64 (table + running sum); a transformation with an infeasible
kernel nothing per kernel and no totals (R4: its total is +inf, N7).  Per
candidate: fp64 iters*t_iter (1) + t_once (1, run-once kernels only) + t_h2d
+ t_d2h (2) + argmin compare (1).  Per design point (/X = /16 per record):
6 int per kernel (work count), 12 int per array (two byte counts), 3 fp64 +
1 conversion per non-zero transfer.
"""
import pytest


def tally(O, sk, skel, x, n, it):
    rc, link = O.fit_pcie(sk.PAPER_TS, sk.PAPER_TL, sk.PAPER_SL)
    P = O.Problem([skel], sk.FX5600, link)
    ok, f, i, c = P.op_tally_one(x, n, n, it, 16)
    assert ok
    return f, i, c


def test_hotspot_1024(O, sk):
    """App. B.2: S1 HotSpot at 1024^2 (one per-iteration kernel, 3 arrays:
    temp_in and power read, temp_out written and live-out -> 3 transfers).
    W = 2^20 work items.  x = 0 (tpb 64, naive: regs 12): occupancy
    min(8, 12, 10) = 8, D = 128 (a power of two), synch 0 -> S = 0; blocks
    = 16384 >= sat: saturated.  fp64 = (1 + 2 + 1) + (1 + 2 + 1) + 9/16."""
    s = sk.s1_hotspot()
    f, i, c = tally(O, sk, s, 0, 1024, 10)
    assert f == 4 + 4 + 9 / 16
    assert i == 6 / 16 + 2 + 36 / 16
    assert c == 1 + 3 / 16
    # x = 1 (tpb 64, smem variant: synch 1, smem 384 B) -> S != 0, D = 128:
    # fp64 per kernel 1 + 2 (S rep + add) + 2 + 1 = 6
    f, i, c = tally(O, sk, s, 1, 1024, 10)
    assert f == 6 + 4 + 9 / 16
    # x = 4 (tpb 128, naive): occupancy min(8, 6, 5) = 5, D = 80 (not a power
    # of two), S = 0 -> 2 (rep) + 1 + 2 + 1 = 6
    f, i, c = tally(O, sk, s, 4, 1024, 10)
    assert f == 6 + 4 + 9 / 16
    # x = 14 (tpb 512, coarse2: regs 20 * 512 > 8192): infeasible -> no
    # kernel arithmetic, no conversion of its block count, and (R4: its total
    # is +inf, outside the argmin, N7) no totals: only the design point's share
    f, i, c = tally(O, sk, s, 14, 1024, 10)
    assert f == 9 / 16
    assert i == 6 / 16 + 36 / 16
    assert c == 3 / 16


def test_stencil_64_below_saturation(O, sk):
    """App. B.1: S0 at 64^2, W = 62^2 = 3844 per kernel (2 kernels), arrays A
    (H2D 16384 B, D2H 15376 B) and B (H2D 1008 B, temporary) -> 3 transfers.
    x = 0: ipb 64 -> 61 blocks < sat = max(16, 7 * 16 + 1) = 113: below
    saturation, tabulated -> 1 fp64 + 2 int per kernel."""
    s = sk.s0_stencil2()
    f, i, c = tally(O, sk, s, 0, 64, 1)
    assert f == 2 * 1 + 4 + 9 / 16
    assert i == 2 * (6 / 16 + 2) + 24 / 16
    assert c == 3 / 16
    # x = 14 infeasible: nothing per kernel
    f, i, c = tally(O, sk, s, 14, 64, 1)
    assert f == 9 / 16 and i == 2 * 6 / 16 + 24 / 16


def test_run_once_kernel_adds_t_once(O, sk):
    """CFD (S4) has a run-once initialisation kernel: the total adds t_once
    (one more fp64 add per candidate than an all-per-iteration skeleton)."""
    s = sk.s4_cfd()
    rc, link = O.fit_pcie(sk.PAPER_TS, sk.PAPER_TL, sk.PAPER_SL)
    P = O.Problem([s], sk.FX5600, link)
    ok, f, i, c = P.op_tally_one(0, 1 << 20, 1, 5, 16)
    assert ok
    # 5 kernels, the record's usage: f - per-kernel part - usage part = 5
    per_kernel = 0.0
    for k in range(5):
        t, reg = O.kernel_time(s, sk.FX5600, 0, k, 1 << 20, 1)
        assert reg in (1, 2, 3, 4)    # every kernel runs (saturated at 2^20 elements)
    h, d = O.usage(s, 1 << 20, 1)
    n_tr = int((h > 0).sum() + (d > 0).sum())
    assert (f - 3 * n_tr / 16) % 1 == 0
    assert f - 3 * n_tr / 16 - 5 * 4 >= 5   # totals 5 (with t_once) + extra terms


def test_invalid_and_batch_mean(O, sk):
    import numpy as np
    s = sk.s1_hotspot()
    rc, link = O.fit_pcie(sk.PAPER_TS, sk.PAPER_TL, sk.PAPER_SL)
    P = O.Problem([s], sk.FX5600, link)
    ok, f, i, c = P.op_tally_one(99 << 16, 64, 64, 1, 16)
    assert not ok and f == i == c == 0.0
    rec = {"skx": np.array([0, 14, 99 << 16], np.uint32), "nx": np.full(3, 1024, np.uint32),
           "ny": np.full(3, 1024, np.uint32), "iters": np.full(3, 10, np.uint32)}
    m = P.op_tally(rec)
    assert m["n_valid"] == 2
    assert m["fp64"] == ((8 + 9 / 16) + 9 / 16) / 2
