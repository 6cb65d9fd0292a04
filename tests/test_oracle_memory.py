"""NEXT-4: pinned vs pageable memory with allocation overhead,
DESIGN.md reading 17.  The paper only names the tradeoff ("explore
the tradeoff between the two types of memory", "account for the
overhead of memory allocation"), so the oracle is pinned to closed forms of
the reading — the crossover size of a linear cost difference, the paper's
Fig. 3 observation as a configured case, degenerate cases — and the
library's host function is checked bitwise against it."""
import math

import numpy as np
import pytest

from paper_conf_ipps_boyermk13_b200 import grophecy as G


def L(O, alpha, beta):
    return O.Link(alpha, beta)


def test_no_transfer_costs_nothing(O):
    z = L(O, 1e-5, 1e-9)
    rc, tp, tg, m = O.choose_memory(z, z, z, z, L(O, 1e-3, 1e-9), 0, 0, 1 << 20)
    assert (rc, tp, tg, m) == (0, 0.0, 0.0, 0)   # tie -> pinned, no allocation


def test_free_allocation_faster_links_pick_pinned(O):
    pin, page, free = L(O, 1e-5, 1e-11), L(O, 2e-5, 5e-11), L(O, 0.0, 0.0)
    for h, d in ((1, 0), (0, 1), (1 << 20, 1 << 10), (1 << 30, 1 << 30)):
        rc, tp, tg, m = O.choose_memory(pin, pin, page, page, free, h, d, 1 << 31)
        assert rc == 0 and m == 0 and tp < tg


def test_expensive_allocation_picks_pageable(O):
    pin, page = L(O, 1e-5, 1e-11), L(O, 2e-5, 5e-11)
    rc, tp, tg, m = O.choose_memory(pin, pin, page, page, L(O, 1.0, 0.0), 1 << 20, 0, 1 << 20)
    assert rc == 0 and m == 1 and tp > 1.0 > tg


def test_crossover_is_the_root_of_the_linear_difference(O):
    """One direction, footprint = transfer size d: pinned - pageable =
    (a_A + a_pin - a_pg) + (b_A + b_pin - b_pg) d, so the choice flips at
    d* = (a_A + a_pin - a_pg) / (b_pg - b_pin - b_A)."""
    a_pin, b_pin = 10e-6, 1 / 55e9
    a_pg, b_pg = 8e-6, 1 / 20e9
    a_A, b_A = 200e-6, 1 / 40e9
    d_star = (a_A + a_pin - a_pg) / (b_pg - b_pin - b_A)
    pin, page, al = L(O, a_pin, b_pin), L(O, a_pg, b_pg), L(O, a_A, b_A)
    lo, hi = int(d_star * 0.99), int(d_star * 1.01) + 1
    assert O.choose_memory(pin, pin, page, page, al, lo, 0, lo)[3] == 1   # below: pageable
    assert O.choose_memory(pin, pin, page, page, al, hi, 0, hi)[3] == 0   # above: pinned
    # and the flip is monotone over a sweep
    ms = [O.choose_memory(pin, pin, page, page, al, 1 << e, 0, 1 << e)[3] for e in range(0, 31)]
    assert ms == sorted(ms, reverse=True)


def test_paper_fig3_small_h2d_prefers_pageable(O):
    """"With the exception of CPU-to-GPU transfers smaller than 2KB, a
    transfer using pinned memory is always faster": links with that property
    (no allocation cost, as in the paper's comparison) reproduce it."""
    a_pg = 5e-6
    b_pg = 1 / 2.0e9
    b_pin = 1 / 2.5e9
    a_pin = a_pg + (b_pg - b_pin) * 2048            # equal at exactly 2 KiB
    pin, page, free = L(O, a_pin, b_pin), L(O, a_pg, b_pg), L(O, 0.0, 0.0)
    for s in (1, 64, 1024, 2000):
        assert O.choose_memory(pin, pin, page, page, free, s, 0, s)[3] == 1
    for s in (2100, 4096, 1 << 20, 1 << 29):
        assert O.choose_memory(pin, pin, page, page, free, s, 0, s)[3] == 0


def test_rejects_footprint_below_transfer(O):
    z = L(O, 1e-5, 1e-9)
    assert O.choose_memory(z, z, z, z, z, 10, 0, 9)[0] == -1
    m = G.MemoryModel()
    with pytest.raises(G.GrophecyError):
        G.choose_memory(m, 0, 10, 9)


def test_library_matches_oracle_bitwise(O):
    """The product's host function (grophecy_choose_memory) vs the oracle on
    random models and sizes, both results and choices."""
    r = np.random.default_rng(17)
    for _ in range(3000):
        p = [(float(r.uniform(0, 5e-5)), float(1 / r.uniform(1e9, 6e10))) for _ in range(5)]
        if r.random() < 0.1:
            p[4] = (0.0, 0.0)
        h, d = (int(x) if r.random() < 0.85 else 0 for x in r.integers(1, 1 << 31, 2))
        fp = max(h, d) + int(r.integers(0, 1 << 31))
        m = G.MemoryModel()
        (m.pinned.h2d.alpha_s, m.pinned.h2d.beta_s_per_byte) = p[0]
        (m.pinned.d2h.alpha_s, m.pinned.d2h.beta_s_per_byte) = p[1]
        (m.pageable.h2d.alpha_s, m.pageable.h2d.beta_s_per_byte) = p[2]
        (m.pageable.d2h.alpha_s, m.pageable.d2h.beta_s_per_byte) = p[3]
        (m.pin_alloc.alpha_s, m.pin_alloc.beta_s_per_byte) = p[4]
        c = G.choose_memory(m, h, d, fp)
        rc, tp, tg, mm = O.choose_memory(*[L(O, *q) for q in p], h, d, fp)
        assert rc == 0
        assert (c.t_pinned_s, c.t_pageable_s, c.memory) == (tp, tg, mm)
        assert not math.isnan(tp) and not math.isnan(tg)


def _problem(O, skels):
    from synth import skeletons as S
    return O.Problem(skels, S.FX5600, O.fit_pcie(1e-5, 1.0, 1 << 20)[1])


def test_eval_mem_reduces_to_the_paper_model(O):
    """Pageable links equal to the pinned ones and a free allocation: every
    array ties, stays pinned, and the projection is the paper's one with the
    pinned links — bitwise."""
    from synth import records as R
    c = R.config("c4")
    idx = np.arange(0, 10**9, 10**9 // 3000, dtype=np.uint64)
    rec = R.gen_records_at(c, idx)
    pin = L(O, 1.0e-5, 4.0e-10)
    P = _problem(O, c["skeletons"])
    P.hl = pin
    P.dl = pin
    for k in range(len(idx)):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, h, d, t, th, td = P.eval_mem_one((pin, pin, pin, pin, L(O, 0.0, 0.0)), *a)
        ok2, h2, d2, t2 = P.eval_one(*a)
        assert (ok, h, d) == (ok2, h2, d2)
        assert np.float64(t).view(np.uint64) == np.float64(t2).view(np.uint64)


def test_eval_mem_expensive_allocation_is_all_pageable(O):
    """A prohibitive allocation: every array pageable, i.e. the paper's model
    with the pageable links."""
    from synth import records as R
    c = R.config("c3")
    rec = R.gen_records(c, 0, 2000)
    pin, page = L(O, 1.0e-5, 2.0e-11), L(O, 2.0e-5, 9.0e-11)
    P = _problem(O, c["skeletons"])
    P.hl = page
    P.dl = page
    for k in range(0, 2000, 3):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, h, d, t, th, td = P.eval_mem_one((pin, pin, page, page, L(O, 1e3, 0.0)), *a)
        assert (ok, h, d, t) == P.eval_one(*a)


def test_eval_mem_hand_case(O):
    """One array read (4 MiB, footprint 4 MiB) and written back: the chosen
    memory and the two terms follow reading 17 by hand."""
    from tests.tiny import DUMMY_KX
    sk = {"name": "h", "arrays": [{"name": "a", "rows": (1, 0, 0, 0), "cols": (0, 8, 0, 0),
                                   "elem_bytes": 4, "liveout": True}],
          "kernels": [{"name": "k", "work": (0, 0, 0, 0), "per_iter": True}],
          "regions": [{"kernel": 0, "array": 0, "mode": "RW", "whole": False, "r0": (0, 0, 0, 0),
                       "r1": (1, 0, 0, 0), "c0": (0, 0, 0, 0), "c1": (0, 8, 0, 0)}],
          "kx": [[DUMMY_KX]]}
    n = 1 << 20
    B = 4 * n
    pin, page = L(O, 1e-5, 1e-10), L(O, 1e-5, 4e-10)
    P = _problem(O, [sk])
    for alloc, want in ((L(O, 1e-4, 0.0), 0), (L(O, 1e-2, 0.0), 1)):
        ok, h, d, t, th, td = P.eval_mem_one((pin, pin, page, page, alloc), 0, n, 1, 1)
        assert ok and (h, d) == (B, B)
        pinned = (alloc.alpha + (1e-5 + 1e-10 * B)) + (1e-5 + 1e-10 * B)
        pageable = (1e-5 + 4e-10 * B) + (1e-5 + 4e-10 * B)
        assert (pinned <= pageable) == (want == 0)
        if want == 0:
            assert th == alloc.alpha + (1e-5 + 1e-10 * B) and td == 1e-5 + 1e-10 * B
        else:
            assert th == 1e-5 + 4e-10 * B and td == 1e-5 + 4e-10 * B
