"""Oracle pins: candidate totals and the argmin.

* Total GPU time = kernels + transfers: with a zero-cost PCIe
  link the total equals the kernel time; with zero work it equals the
  transfer time built from per-array transfers.
* Transfers happen once; per-iteration kernels repeat: the kernel
  part is exactly linear in ``iters``; run-once kernels are not multiplied.
* Best = argmin over (t, global index), ties to the lowest index, checked
  against Python's min() over the oracle's own per-candidate outputs.
"""
import math

import numpy as np
import pytest

from synth import records as R


ZERO_LINK = None


@pytest.fixture(scope="module")
def zlink(O):
    rc, l = O.fit_pcie(0.0, 1e-300, 1)
    l.alpha = 0.0
    l.beta = 0.0
    return l


def test_total_is_kernel_time_without_transfers(O, sk, zlink):
    s = sk.s0_stencil2()
    P = O.Problem([s], sk.FX5600, zlink)
    for x in range(16):
        ok, h, d, t = P.eval_one(x, 64, 64, 1)
        t0, _ = O.kernel_time(s, sk.FX5600, x, 0, 64, 64)
        t1, _ = O.kernel_time(s, sk.FX5600, x, 1, 64, 64)
        assert ok and t == t0 + t1


def test_total_is_transfer_time_without_work(O, sk, paper_link):
    """S0 at 2x2: (nx-2)(ny-2) = 0 work items -> kernel time 0; A (4 el) read
    whole by k0, B (4 el) read whole by k1, interiors empty -> two 16-byte
    transfers in, none out: t = (0 + T(16)) + T(16) = 2*T(16) exactly."""
    P = O.Problem([sk.s0_stencil2()], sk.FX5600, paper_link)
    ok, h, d, t = P.eval_one(3, 2, 2, 5)
    assert ok and h == 32 and d == 0
    assert t == 2 * (1e-5 + 16 * 4e-10)


def test_iters_scale_kernels_only(O, sk, zlink, paper_link):
    """with free transfers, t(iters) = iters * t(1) for an all-per-iter
    skeleton (exact for iters = 2^k); with the paper link, the transfer part
    does not grow."""
    P = O.Problem([sk.s1_hotspot()], sk.FX5600, zlink)
    for x in (0, 5, 13):
        _, _, _, t1 = P.eval_one(x, 1024, 1024, 1)
        for it in (2, 8, 1024):
            _, _, _, ti = P.eval_one(x, 1024, 1024, it)
            assert ti == it * t1
    Q = O.Problem([sk.s1_hotspot()], sk.FX5600, paper_link)
    _, h1, d1, _ = Q.eval_one(0, 1024, 1024, 1)
    _, h9, d9, _ = Q.eval_one(0, 1024, 1024, 9)
    assert (h1, d1) == (h9, d9) == (8 << 20, 4 << 20)


def test_run_once_kernel_not_multiplied(O, sk, zlink):
    """CFD's initialisation kernel runs once (P:L167 reading 12):
    t(iters) - t(1) == (iters-1) * t_iter for per-iteration kernels only."""
    s = sk.s4_cfd()
    P = O.Problem([s], sk.FX5600, zlink)
    nx = 97000
    t_once, _ = O.kernel_time(s, sk.FX5600, 0, 0, nx, 1)
    t_iter = 0.0
    for k in range(1, 5):
        t_iter = t_iter + O.kernel_time(s, sk.FX5600, 0, k, nx, 1)[0]
    _, _, _, t4 = P.eval_one(0, nx, 1, 4)
    assert t_once > 0 and t_iter > 0
    assert t4 == t_once + 4.0 * t_iter


def test_infeasible_candidate_is_infinite(O, sk, paper_link):
    P = O.Problem([sk.s0_stencil2()], sk.FX5600, paper_link)
    ok, h, d, t = P.eval_one(14, 64, 64, 1)   # 512 threads x 20 regs > 8192
    assert ok and math.isinf(t) and (h, d) == (17392, 15376)


@pytest.mark.parametrize("rec", [(1 << 16, 64, 64, 1), (16, 64, 64, 1), (0, 0, 64, 1),
                                 (0, 64, 0, 1), (0, (1 << 20) + 1, 64, 1), (0, 64, 64, 0)])
def test_invalid_records(O, sk, paper_link, rec):
    P = O.Problem([sk.s0_stencil2()], sk.FX5600, paper_link)
    ok, h, d, t = P.eval_one(*rec)
    assert not ok and h == 0 and d == 0 and math.isnan(t)


def test_max_sizes_are_valid(O, sk, paper_link):
    P = O.Problem([sk.s1_hotspot()], sk.FX5600, paper_link)
    ok, h, d, t = P.eval_one(0, 1 << 20, 1 << 20, 1)
    assert ok and h == 8 << 40 and d == 4 << 40 and math.isfinite(t)


def _brute_best(h, d, t, base=0):
    cands = [(t[i], base + i) for i in range(len(t)) if math.isfinite(t[i])]
    if not cands:
        return None
    return min(cands)


@pytest.mark.parametrize("cfg", ["c1", "c2"])
def test_best_is_brute_force_min(O, paper_link, cfg, sk):
    c = R.config(cfg)
    c = R.with_n(c, min(c["n"], 20000))
    rec = R.gen_records(c)
    P = O.Problem(c["skeletons"], sk.FX5600, paper_link)
    h, d, t = P.eval(rec)
    for base in (0, 123456789):
        rc, b = P.best(rec, index_base=base)
        tb, ib = _brute_best(h, d, t, base)
        assert rc == 0 and b.t_total_s == tb and b.index == ib
        assert b.h2d_bytes == h[ib - base] and b.d2h_bytes == d[ib - base]


def test_best_c1_is_xform5(O, sk, paper_link):
    """C1: the winner among the 16 stencil transformations."""
    c = R.config("c1")
    P = O.Problem(c["skeletons"], sk.FX5600, paper_link)
    rc, b = P.best(R.gen_records(c))
    assert rc == 0 and b.index == 5


def test_best_ties_go_to_lowest_index(O, sk, paper_link):
    """Exact ties happen: HotSpot at 1024^2 with 10 iterations has transformations
    with bitwise-equal totals; duplicates of one record tie by construction."""
    P = O.Problem([sk.s1_hotspot()], sk.FX5600, paper_link)
    rec = {k: np.array(v, np.uint32) for k, v in
           {"skx": [5, 3, 5, 5], "nx": [1024] * 4, "ny": [1024] * 4, "iters": [10] * 4}.items()}
    h, d, t = P.eval(rec)
    assert t[0] == t[2] == t[3]
    rc, b = P.best(rec)
    assert b.index == (0 if t[0] <= t[1] else 1)
    rec2 = {k: v[[1, 0, 2, 3]] for k, v in rec.items()}
    _, b2 = P.best(rec2, index_base=10)
    assert b2.index == (11 if t[0] <= t[1] else 10)
    # equal-time transformations in the library (no bias by transformation id)
    tt = [P.eval_one(x, 1024, 1024, 10)[3] for x in range(16)]
    groups = {}
    for x, v in enumerate(tt):
        groups.setdefault(v, []).append(x)
    ties = [g for g in groups.values() if len(g) > 1]
    assert ties, "expected exact ties among HotSpot transformations"
    for g in ties:
        rec3 = {"skx": np.array(g[::-1], np.uint32), "nx": np.full(len(g), 1024, np.uint32),
                "ny": np.full(len(g), 1024, np.uint32), "iters": np.full(len(g), 10, np.uint32)}
        _, b3 = P.best(rec3)
        if math.isfinite(tt[g[0]]):
            assert b3.index == 0


def test_best_all_invalid_or_infeasible(O, sk, paper_link):
    P = O.Problem([sk.s0_stencil2()], sk.FX5600, paper_link)
    rec = {"skx": np.array([14, 14, 99], np.uint32), "nx": np.array([64, 64, 64], np.uint32),
           "ny": np.array([64, 64, 64], np.uint32), "iters": np.array([1, 1, 1], np.uint32)}
    rc, b = P.best(rec)
    assert rc != 0 and b.index == 2**64 - 1 and b.n_invalid == 1 and b.n_valid == 2


def test_threads_do_not_change_results(O, sk, paper_link):
    c = R.with_n(R.config("c2"), 5000)
    rec = R.gen_records(c)
    P = O.Problem(c["skeletons"], sk.FX5600, paper_link)
    a = P.eval(rec, nthreads=1)
    b = P.eval(rec, nthreads=7)
    for x, y in zip(a, b):
        assert np.array_equal(x, y)
    r1, b1 = P.best(rec, nthreads=1)
    r7, b7 = P.best(rec, nthreads=7)
    assert (b1.index, b1.t_total_s) == (b7.index, b7.t_total_s)
