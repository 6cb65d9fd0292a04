"""Oracle pins for the NEXT-1/NEXT-2 rows:
* time components: t == ((t_once + iters * t_iter) + t_h2d) + t_d2h bitwise,
  and the kernel-only / transfer-only predictors of Table II;
* best transformation per group against Python's groupby + min over
  the oracle's own per-candidate outputs;
* the product's host speedup helpers against the oracle's (which are pinned
  to Table II arithmetic in test_oracle_validation.py)."""
import itertools
import math

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S


@pytest.fixture(scope="module")
def P4(O, paper_link):
    c = R.config("c4")
    return c, O.Problem(c["skeletons"], S.FX5600, paper_link)


def test_parts_compose_to_total(O, P4):
    c, P = P4
    idx = np.arange(0, 10**9, 10**9 // 3000, dtype=np.uint64)
    rec = R.gen_records_at(c, idx)
    for k in range(len(idx)):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, h, d, t = P.eval_one(*a)
        ok2, (ti, to, th, td) = P.eval_parts_one(*a)
        assert ok and ok2
        assert t == ((to + a[3] * ti) + th) + td
        # transfer part depends only on the usage; kernel part scales with iters
        ok3, (ti3, to3, th3, td3) = P.eval_parts_one(a[0], a[1], a[2], 7)
        assert (ti3, to3, th3, td3) == (ti, to, th, td)


def test_parts_invalid_are_nan(O, P4):
    c, P = P4
    ok, parts = P.eval_parts_one(0, 0, 5, 1)
    assert not ok and all(math.isnan(v) for v in parts)


def _brute_groups(P, rec, base=0):
    n = len(rec["skx"])
    keys = [((int(rec["skx"][i]) >> 16), int(rec["nx"][i]), int(rec["ny"][i]), int(rec["iters"][i]))
            for i in range(n)]
    out = []
    i = 0
    for k, grp in itertools.groupby(range(n), key=lambda j: keys[j]):
        g = list(grp)
        cands = []
        for j in g:
            ok, h, d, t = P.eval_one(*[int(rec[f][j]) for f in ("skx", "nx", "ny", "iters")])
            if ok and math.isfinite(t):
                cands.append((t, base + j))
        best = min(cands) if cands else (math.inf, 2**64 - 1)
        out.append((base + g[0], len(g), best[1], best[0]))
    return out


def test_group_best_is_groupby_min(O, P4):
    c, P = P4
    rng = np.random.default_rng(3)
    for trial in range(5):
        # runs of random lengths over a few points, some invalid / infeasible records
        rec = {k: [] for k in ("skx", "nx", "ny", "iters")}
        while len(rec["skx"]) < 600:
            s = int(rng.integers(0, 16))
            L = int(rng.integers(1, 40))
            n0 = int(rng.choice([64, 300, 1024, 4000]))
            it = int(rng.integers(1, 4))
            for _ in range(L):
                x = int(rng.integers(0, 17))   # 16 is an invalid transformation
                rec["skx"].append((s << 16) | x)
                rec["nx"].append(n0)
                rec["ny"].append(n0 if s not in (4, 5) else 1)
                rec["iters"].append(it)
        rec = {k: np.array(v, np.uint32) for k, v in rec.items()}
        want = _brute_groups(P, rec, base=11)
        f, cnt, bi, bt = P.group_best(rec, index_base=11)
        got = list(zip(f.tolist(), cnt.tolist(), bi.tolist(), bt.tolist()))
        assert len(got) == len(want)
        for g, w in zip(got, want):
            assert g[:3] == w[:3] and (g[3] == w[3])


def test_group_best_c1_single_group(O, paper_link):
    c = R.config("c1")
    P = O.Problem(c["skeletons"], S.FX5600, paper_link)
    f, cnt, bi, bt = P.group_best(R.gen_records(c))
    assert list(f) == [0] and list(cnt) == [16] and list(bi) == [5]


def test_product_speedup_helpers_match_oracle(O):
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy as G
    rng = np.random.default_rng(8)
    for _ in range(2000):
        a, b = float(rng.uniform(1e-6, 10)), float(rng.uniform(1e-6, 10))
        assert G.speedup(a, b) == O.speedup(a, b)
        assert G.error_magnitude(a, b) == O.error_magnitude(a, b)
    # Table II, Stassuij
    assert round(100 * G.error_magnitude(1.10, 0.39)) == 182


def _exact_first_win(ti, to, th, td, c, limit=10**6):
    """Brute force over integer iteration counts in exact rational arithmetic:
    the smallest it >= 1 with F + it * t_iter < it * c (GPU strictly faster)."""
    from fractions import Fraction as Fr
    F = Fr(to) + Fr(th) + Fr(td)
    for it in range(1, limit):
        if F + it * Fr(ti) < it * Fr(c):
            return it
    return None


def test_crossover_closed_form_and_brute_force(O):
    """NEXT-2 break-even iteration count: a hand case, then dyadic inputs
    (every sum and the quotient exact) against a brute-force scan of the
    definition in exact arithmetic."""
    # F = (1 + 0.5) + 0.5 = 2, c - t_iter = 1: break-even at 2 iterations,
    # GPU strictly faster from 3 on
    assert O.crossover(1.0, 1.0, 0.5, 0.5, 2.0) == (2.0, 3)
    # GPU never wins
    assert O.crossover(2.0, 1.0, 0.0, 0.0, 2.0) == (math.inf, 2**64 - 1)
    assert O.crossover(3.0, 0.0, 0.0, 0.0, 2.0) == (math.inf, 2**64 - 1)
    # no one-time cost: the first iteration already wins
    assert O.crossover(1.0, 0.0, 0.0, 0.0, 2.0) == (0.0, 1)
    # invalid (NaN) inputs
    v, m = O.crossover(math.nan, 1.0, 1.0, 1.0, 2.0)
    assert math.isnan(v) and m == 2**64 - 1
    rng = np.random.default_rng(5)
    for _ in range(400):
        ti = int(rng.integers(0, 64)) / 64.0
        to, th, td = (int(rng.integers(0, 4096)) / 64.0 for _ in range(3))
        c = ti + 2.0 ** -int(rng.integers(0, 6))          # c - t_iter a power of two: exact quotient
        v, m = O.crossover(ti, to, th, td, c)
        want = _exact_first_win(ti, to, th, td, c)
        assert m == want, (ti, to, th, td, c, v)
    # huge break-even counts saturate instead of wrapping
    v, m = O.crossover(0.0, 2.0 ** 70, 0.0, 0.0, 1.0)
    assert v == 2.0 ** 70 and m == 2**64 - 1
    v, m = O.crossover(0.0, 2.0 ** 60, 0.0, 0.0, 1.0)
    assert m == 2**60 + 1
