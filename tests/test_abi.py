"""The C-ABI boundary on CPU: the library loads, exports every symbol
include/grophecy.h declares, and its host-only entry points behave
(no compute calls need a GPU here)."""
import math
import os
import re

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def G():
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy
    return grophecy


def header_functions():
    src = open(os.path.join(ROOT, "include", "grophecy.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(grophecy_[a-z_0-9]+)\s*\(", src)))


def test_every_declared_symbol_is_exported(G):
    import ctypes
    lib = ctypes.CDLL(G.LIB_PATH)
    names = header_functions()
    assert len(names) >= 18
    for n in names:
        assert hasattr(lib, n), n
    assert set(names) == set(G.EXPORTED)


def test_abi_version(G):
    assert G.lib().grophecy_abi_version() == G.ABI_VERSION == 4


def test_fit_pcie_matches_oracle_bitwise(G, O):
    rng = np.random.default_rng(5)
    for _ in range(2000):
        tS = float(rng.uniform(0, 1e-3))
        tL = float(rng.uniform(1e-4, 1.0))
        sL = int(rng.integers(1, 1 << 40))
        a = G.fit_pcie(tS, tL, sL)
        rc, b = O.fit_pcie(tS, tL, sL)
        assert rc == 0 and a.alpha_s == b.alpha and a.beta_s_per_byte == b.beta
        for d in (0, 1, int(rng.integers(1, 1 << 45))):
            assert G.pcie_time(a, d) == O.pcie_time(b, d)


@pytest.mark.parametrize("args", [(-1e-6, 1.0, 10), (1e-6, 0.0, 10), (1e-6, 1.0, 0),
                                  (math.nan, 1.0, 10), (1e-6, math.inf, 10)])
def test_fit_pcie_rejects(G, args):
    with pytest.raises(G.GrophecyError) as e:
        G.fit_pcie(*args)
    assert e.value.code == G.EINVAL


def test_validate_accepts_library(G):
    for c in ("c1", "c2", "c3", "c4"):
        assert G.validate(R.config(c)["skeletons"], S.FX5600) == G.OK


def _s0():
    return S.s0_stencil2()


@pytest.mark.parametrize("mutate,code", [
    (lambda s: s["kernels"].clear(), -1),
    (lambda s: s["regions"].append(dict(s["regions"][0], kernel=5)), -1),
    (lambda s: s["regions"].append(dict(s["regions"][0], array=7)), -1),
    (lambda s: s["regions"].append(dict(s["regions"][0], r_step=65)), -2),
    (lambda s: s["regions"].extend([dict(s["regions"][0], array=0, whole=False, c_step=7),
                                    dict(s["regions"][0], array=0, whole=False, c_step=11)]), -2),
    (lambda s: s["regions"].extend([dict(s["regions"][1])] * 40), -2),
    (lambda s: s["arrays"].extend([dict(s["arrays"][0])] * 20), -2),
    (lambda s: s["kernels"].__setitem__(0, dict(s["kernels"][0], work=(0, 1 << 16, 0, 0))), -2),
    (lambda s: s["kx"][0].__setitem__(0, dict(s["kx"][0][0], total=1.0)), -1),
    (lambda s: s["kx"][0].__setitem__(0, dict(s["kx"][0][0], tpb=0)), -2),
    (lambda s: s["kx"][0].__setitem__(0, dict(s["kx"][0][0], upm=0.5)), -1),
    (lambda s: s["kx"][0].__setitem__(0, dict(s["kx"][0][0], coal=math.nan)), -1),
])
def test_validate_rejects(G, mutate, code):
    s = _s0()
    mutate(s)
    assert G.validate([s], S.FX5600) == code


def test_validate_rejects_bad_gpu(G):
    g = dict(S.FX5600, freq_hz=0.0)
    assert G.validate([_s0()], g) == G.EINVAL
    g = dict(S.FX5600, n_sm=0)
    assert G.validate([_s0()], g) == G.EINVAL


def test_combine_host_is_minloc(G):
    rng = np.random.default_rng(9)
    for _ in range(300):
        k = int(rng.integers(0, 9))
        res = []
        for _ in range(k):
            if rng.random() < 0.2:
                res.append(G.BestResult(math.inf, G.UINT64_MAX, 0, 0, int(rng.integers(0, 5)),
                                        int(rng.integers(0, 5))))
            else:
                t = float(rng.choice([1.0, 2.0, 0.5, 3.25]))
                res.append(G.BestResult(t, int(rng.integers(0, 100)), int(rng.integers(0, 9)),
                                        int(rng.integers(0, 9)), int(rng.integers(0, 5)),
                                        int(rng.integers(1, 5))))
        out = G.best_combine_host(res)
        valid = [(r.t_total_s, r.index, r.h2d_bytes, r.d2h_bytes) for r in res
                 if r.index != G.UINT64_MAX]
        assert out.n_invalid == sum(r.n_invalid for r in res)
        assert out.n_valid == sum(r.n_valid for r in res)
        if not valid:
            assert out.index == G.UINT64_MAX and math.isinf(out.t_total_s)
        else:
            best = min(valid, key=lambda v: (v[0], v[1]))
            assert (out.t_total_s, out.index) == best[:2]
            # the winner's byte counts travel with it (first occurrence of the min)
            cand = [v for v in valid if (v[0], v[1]) == best[:2]]
            assert (out.h2d_bytes, out.d2h_bytes) in [(v[2], v[3]) for v in cand]


def test_no_gpu_fails_loudly(G):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(G.GrophecyError) as e:
        G.Space([_s0()], S.FX5600, device=0)
    assert e.value.code == G.ECUDA


def _check_plan(G, O, s, sizes):
    covered = 0
    for nx, ny in sizes:
        rc, h, d, tx, ty = G.plan_usage_host(s, nx, ny)
        if rc != G.OK:
            assert rc == G.ELIMIT and (nx < tx or ny < ty or tx == 0xFFFFFFFF)
            continue
        covered += 1
        oh, od = O.usage(s, nx, ny)
        assert list(h) == [int(v) for v in oh], (s["name"], nx, ny)
        assert list(d) == [int(v) for v in od], (s["name"], nx, ny)
    return covered


def test_usage_plans_match_oracle_library(G, O):
    """The compiled usage plans (closed-form band programs the kernel runs)
    reproduce the oracle's data usage at every size of their domain."""
    r = np.random.default_rng(17)
    sizes = [(int(a), int(b)) for a, b in zip(np.exp2(r.uniform(0, 20, 120)).astype(int),
                                                 np.exp2(r.uniform(0, 20, 120)).astype(int))]
    sizes += [(1, 1), (2, 2), (3, 5), (1 << 20, 1 << 20), (1 << 20, 1), (1, 1 << 20)]
    skels = [f() for f in S.LIBRARY] + S.random_skeletons(0x5EED0003, 20)
    tot = 0
    for s in skels:
        tot += _check_plan(G, O, s, sizes)
    assert tot > 0.5 * len(sizes) * len(skels)


def test_usage_plans_match_oracle_random_tiny(G, O):
    from tests.tiny import random_tiny_skeleton, rng
    r = rng(555)
    tot = 0
    for _ in range(400):
        s, _, _ = random_tiny_skeleton(r)
        sizes = [(int(r.integers(1, 2000)), int(r.integers(1, 2000))) for _ in range(6)]
        sizes += [(1 << 20, 1 << 20), (int(r.integers(1, 64)), 1 << 20)]
        tot += _check_plan(G, O, s, sizes)
    assert tot > 500


def test_group_merge_host_rules():
    from paper_conf_ipps_boyermk13_b200 import grophecy as G
    NONE = 2**64 - 1
    a = G.GroupResult(2.0, 10, 5, 12, 100, 50)
    b = G.GroupResult(1.0, 15, 3, 16, 7, 8)
    m = G.group_merge_host(a, b)
    assert (m.best_t_s, m.first, m.count, m.best_index, m.h2d_bytes, m.d2h_bytes) == \
        (1.0, 10, 8, 16, 7, 8)
    # tie: the lower index (a's) wins
    b2 = G.GroupResult(2.0, 15, 3, 16, 7, 8)
    m = G.group_merge_host(a, b2)
    assert (m.best_index, m.h2d_bytes) == (12, 100)
    # "none" halves never win
    na = G.GroupResult(float("inf"), 10, 5, NONE, 0, 0)
    m = G.group_merge_host(na, b)
    assert (m.best_index, m.count) == (16, 8)
    m = G.group_merge_host(b, G.GroupResult(float("inf"), 18, 2, NONE, 0, 0))
    assert (m.best_index, m.first, m.count) == (16, 15, 5)
    # b must follow a
    with pytest.raises(G.GrophecyError):
        G.group_merge_host(a, G.GroupResult(1.0, 16, 3, 16, 7, 8))


def test_usage_plans_with_maywrites_match_oracle(G, O):
    """Irregular writes (may-writes, reading 10) keep the plan path; its
    closed forms reproduce the oracle."""
    from tests.tiny import random_tiny_skeleton, rng
    r = rng(556)
    tot = 0
    for _ in range(300):
        s, _, _ = random_tiny_skeleton(r, maywrite=True)
        sizes = [(int(r.integers(1, 2000)), int(r.integers(1, 2000))) for _ in range(6)]
        tot += _check_plan(G, O, s, sizes)
    assert tot > 200


def test_strided_and_hull_skeletons_have_no_plan(G):
    """Strided sections and the hull mode take the general device paths."""
    from tests.tiny import random_tiny_skeleton, rng
    r = rng(557)
    n_str = 0
    for _ in range(60):
        s, nx, ny = random_tiny_skeleton(r, strided=True)
        strided = any(g.get("r_step", 1) > 1 or g.get("c_step", 1) > 1
                      for g in s["regions"] if not g["whole"])
        rc, h, d, tx, ty = G.plan_usage_host(s, 64, 64)
        if strided:
            n_str += 1
            assert rc == G.ELIMIT and tx == 0xFFFFFFFF
        rc, h, d, tx, ty = G.plan_usage_host(dict(s, hull=True), 64, 64)
        assert rc == G.ELIMIT and tx == 0xFFFFFFFF
    assert n_str > 20


def test_rank3_skeletons_have_no_plan_and_validate(G):
    """Rank-3 arrays (N4r) take the general sweep: no usage plan; the space
    validation accepts them and rejects out-of-range plane coefficients."""
    from tests.tiny import random_tiny_skeleton, rng
    r = rng(9900)
    for _ in range(50):
        sk, nx, ny = random_tiny_skeleton(r, rank3=True)
        if not any(a.get("planes", (1, 0, 0, 0)) != (1, 0, 0, 0) for a in sk["arrays"]) and \
                not any(g.get("p0", (0, 0, 0, 0)) != (0, 0, 0, 0) for g in sk["regions"]):
            continue
        rc = G.plan_stats(sk)[0]
        assert rc == G.ELIMIT
    sk, _, _ = random_tiny_skeleton(r, rank3=True)
    sk["arrays"][0]["planes"] = (0, 1 << 16, 0, 0)
    from synth import skeletons as S
    assert G.validate([sk], S.FX5600) == G.ELIMIT
