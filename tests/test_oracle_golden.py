"""Oracle pins against values fixed outside the oracle.

* SURVEY.md Appendix B.1 / B.2 golden vectors (``tests/golden/appendix_b.txt``):
  per-transformation totals of config C1 and of HotSpot at 1024^2, including
  the exact ties and the infeasible transformation.  These pin the whole
  composition: data usage + Eq. (1) + our kernel-model
  reading N5 (the paper prints no formula: P:L13, L67) + totals.
* The hand derivation of App. B.1 xform 8 (SURVEY.md §8(c) "What pins each
  part"): blocks = 16, N = 8, rep = 1, case 1, cyc = 4200 + 160 + 16*7 = 4472.
* N2 floor semantics of affine8 against Python's floor division (negative
  numerators round toward -inf), on random coefficients.
* Eq. (1) against exact rational arithmetic: T(d) = RN(alpha + RN(beta*d))
  computed with fractions.Fraction, rounded once per operation (float() of a
  Fraction is correctly rounded).
"""
import math
import os
from fractions import Fraction

import numpy as np
import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


def load_appendix_b():
    rows = {"B1": {}, "B2": {}}
    scal = {}
    for ln in open(os.path.join(HERE, "golden", "appendix_b.txt")):
        ln = ln.split("#")[0].strip()
        if not ln:
            continue
        f = ln.split()
        if f[0] in rows:
            t = math.inf if f[4] == "inf" else float.fromhex(f[4])
            rows[f[0]][int(f[1])] = (int(f[2]), int(f[3]), t)
        else:
            scal[f[0]] = f[1]
    return rows, scal


def test_appendix_b1_c1_every_transformation(O, sk, paper_link):
    rows, scal = load_appendix_b()
    P = O.Problem([sk.s0_stencil2()], sk.FX5600, paper_link)
    assert len(rows["B1"]) == 16
    for x, (h, d, t) in rows["B1"].items():
        ok, oh, od, ot = P.eval_one(x, 64, 64, 1)
        assert ok and (oh, od) == (h, d)
        assert ot == t, (x, ot.hex(), t)
    ok, t_iter, t_once, th, td = (lambda r: (r[0],) + r[1])(P.eval_parts_one(0, 64, 64, 1))
    assert th == float.fromhex(scal["B1_TH2D"]) and td == float.fromhex(scal["B1_TD2H"])
    rec = {"skx": np.arange(16, dtype=np.uint32), "nx": np.full(16, 64, np.uint32),
           "ny": np.full(16, 64, np.uint32), "iters": np.ones(16, np.uint32)}
    rc, b = P.best(rec)
    assert rc == 0 and b.index == int(scal["B1_ARGMIN"])


def test_appendix_b2_hotspot_ties(O, sk, paper_link):
    rows, scal = load_appendix_b()
    P = O.Problem([sk.s1_hotspot()], sk.FX5600, paper_link)
    for x, (h, d, t) in rows["B2"].items():
        ok, oh, od, ot = P.eval_one(x, 1024, 1024, 10)
        assert ok and (oh, od) == (h, d)
        assert ot == t, (x, ot.hex(), t)
    rec = {"skx": np.arange(16, dtype=np.uint32), "nx": np.full(16, 1024, np.uint32),
           "ny": np.full(16, 1024, np.uint32), "iters": np.full(16, 10, np.uint32)}
    rc, b = P.best(rec)
    assert rc == 0 and b.index == int(scal["B2_ARGMIN"])
    # tie-break: the tie set {8, 12, 0} in that order at global indices
    # 100..102 -> the lowest global index wins (100, transformation 8)
    sub = {k: v[[8, 12, 0]] for k, v in rec.items()}
    rc, b = P.best(sub, index_base=100)
    assert b.index == 100 and b.t_total_s == rows["B2"][0][2]


def test_appendix_b1_hand_derivation_xform8(O, sk):
    """xform 8 (tpb 256, naive) at 64^2: W = 62*62 = 3844,
    blocks = ceil(3844/256) = 16, asm = 16, abps = 1, N = 8 warps, rep = 1,
    mwp = min(105, 11.67, 8) = 8, cwp = min(27.25, 8) = 8 -> H&K case 1:
    cyc = Mem_cycles + Comp + (Comp/Mem)(MWP-1) = 4200 + 160 + 16*7 = 4472."""
    t, regime = O.kernel_time(sk.s0_stencil2(), sk.FX5600, 8, 0, 64, 64)
    assert regime == 1
    assert t == 4472.0 / 1.35e9


def test_affine8_floor_matches_python_floor_division(O):
    rng = np.random.default_rng(8)
    for _ in range(2000):
        c = [int(v) for v in rng.integers(-(1 << 15), 1 << 15, 4)]
        nx, ny = (int(v) for v in rng.integers(1, 1 << 20, 2))
        want = c[0] + (c[1] * nx + c[2] * ny + c[3] * nx * ny) // 8   # floor toward -inf
        assert O.affine8(tuple(c), nx, ny) == want
    # the negative-numerator cases by hand: floor(-1/8) = -1, floor(-8/8) = -1,
    # floor(-9/8) = -2
    assert O.affine8((0, -1, 0, 0), 1, 1) == -1
    assert O.affine8((0, -8, 0, 0), 1, 1) == -1
    assert O.affine8((0, -9, 0, 0), 1, 1) == -2
    assert O.affine8((5, 0, 0, -3), 1, 1) == 4


def _rn(fr):
    """Round a Fraction to the nearest binary64 (ties to even): float()."""
    return Fraction(float(fr))


@pytest.mark.parametrize("alpha,beta", [(1e-5, 4e-10), (1.44e-5, 1.0 / 55.5e9),
                                        (7.3e-6, 3.1e-11)])
def test_pcie_time_exact_rational(O, alpha, beta):
    from oracle.oracle import Link
    link = Link(alpha, beta)
    rng = np.random.default_rng(3)
    sizes = [1, 2, 1000, 1 << 10, 12345, 1 << 20, (1 << 29) + 7, 1 << 40] + \
        [int(v) for v in rng.integers(1, 1 << 40, 200)]
    for d in sizes:
        want = float(_rn(Fraction(alpha) + _rn(Fraction(beta) * d)))
        assert O.pcie_time(link, d) == want
    assert O.pcie_time(link, 0) == 0.0
