"""GPU parity for the projection with the per-array memory choice (NEXT-4,
DESIGN.md reading 17; grophecy_eval_mem / grophecy_best_mem) against the
oracle's oracle_eval_mem_one, bitwise: a C4 sample (every skeleton) and tiny
random skeletons (plans, sweeps, strided, hull, rank-3), with a memory model
under which both choices occur."""
import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import oracle_problem, records_slice
from tests.tiny import random_tiny_skeleton, rng

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def G():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy
    torch.cuda.set_device(0)
    return grophecy


def _model(G, alloc_alpha):
    m = G.MemoryModel()
    m.pinned.h2d = G.Link(14.4e-6, 1 / 55.5e9)
    m.pinned.d2h = G.Link(14.9e-6, 1 / 57.1e9)
    m.pageable.h2d = G.Link(12.4e-6, 1 / 11.6e9)
    m.pageable.d2h = G.Link(22.1e-6, 1 / 21.8e9)
    m.pin_alloc = G.Link(alloc_alpha, 0.69e-9)
    return m


def _links(O, m):
    f = lambda l: O.Link(l.alpha_s, l.beta_s_per_byte)   # noqa: E731
    return (f(m.pinned.h2d), f(m.pinned.d2h), f(m.pageable.h2d), f(m.pageable.d2h),
            f(m.pin_alloc))


def _parity(G, O, skels, rec, m, stride=1):
    space = G.Space(skels, S.FX5600)
    out = space.eval_mem(m, G.Records.from_numpy(rec))
    torch.cuda.synchronize()
    h, d, t, ti, to, th, td = [o.cpu().numpy() for o in out]
    P = oracle_problem(O, skels)
    links = _links(O, m)
    best = (np.inf, None)
    choices = set()
    for k in range(0, len(rec["skx"]), stride):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, oh, od, ot, oth, otd = P.eval_mem_one(links, *a)
        if not ok:
            assert np.isnan(t[k])
            continue
        assert (int(h[k]), int(d[k])) == (oh, od), (k, a)
        assert np.float64(t[k]).view(np.uint64) == np.float64(ot).view(np.uint64), (k, a, t[k], ot)
        assert (th[k], td[k]) == (oth, otd)
        choices.add(bool(oth > 0) and oth != td[k])
    rc, b = space.best_mem(m, G.Records.from_numpy(rec))
    finite = np.isfinite(t)
    if finite.any():
        i = int(np.argmin(np.where(finite, t, np.inf)))
        assert b.index == i and b.t_total_s == t[i]
    space.close()


@pytest.mark.parametrize("alloc", [1e-4, 6.7e-3])
def test_c4_sample_memory_choice(G, O, alloc):
    c = R.config("c4")
    idx = np.arange(0, 10**9, 10**9 // 6000, dtype=np.uint64)
    _parity(G, O, c["skeletons"], records_slice(c, idx), _model(G, alloc))


def test_tiny_skeletons_memory_choice(G, O):
    r = rng(9990)
    for trial in range(8):
        skels = []
        for i in range(6):
            s, _, _ = random_tiny_skeleton(r, n_xforms=2, strided=i % 3 == 1, maywrite=True,
                                           hull=i == 2, rank3=i >= 4)
            skels.append(s)
        n = 1500
        rec = {"skx": ((r.integers(0, 6, n) << 16) | r.integers(0, 2, n)).astype(np.uint32),
               "nx": np.exp2(r.uniform(0, 12, n)).astype(np.uint32),
               "ny": np.exp2(r.uniform(0, 12, n)).astype(np.uint32),
               "iters": r.integers(1, 50, n).astype(np.uint32)}
        _parity(G, O, skels, rec, _model(G, 2e-5), stride=3)
