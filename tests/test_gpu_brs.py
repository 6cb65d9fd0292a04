"""GPU parity for the full-BRS row: strided
sections, irregular (may-) writes and the Havlak-Kennedy approximate-UNION
mode, through the C ABI against the oracle, bitwise, on the same seeded
inputs — tiny random skeletons over many sizes (general device paths,
ragged tiles), the C3-shaped strided / hull workloads at prefix sizes and at
full size on sampled outputs, and design spaces that mix the plan, sweep
and hull paths inside one warp tile."""
import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import oracle_problem, paper_pcie, records_slice
from tests.test_gpu_parity import _full_size_check, run_parity
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


@pytest.fixture(scope="module")
def pc(G):
    return paper_pcie(G)


def _tiny_space(r, hull_every=0, n_sk=6):
    skels = []
    for i in range(n_sk):
        s, _, _ = random_tiny_skeleton(r, n_xforms=2, strided=True, maywrite=True,
                                       hull=bool(hull_every) and i % hull_every == 0)
        skels.append(s)
    return skels


def _tiny_records(r, n, n_sk, big=False):
    if big:
        nx = np.exp2(r.uniform(0, 20, n)).astype(np.uint32)
        ny = np.exp2(r.uniform(0, 20, n)).astype(np.uint32)
    else:
        nx = r.integers(1, 40, n).astype(np.uint32)
        ny = r.integers(1, 40, n).astype(np.uint32)
    return {"skx": ((r.integers(0, n_sk, n) << 16) | r.integers(0, 2, n)).astype(np.uint32),
            "nx": nx, "ny": ny, "iters": r.integers(1, 50, n).astype(np.uint32)}


@pytest.mark.parametrize("hull_every", [0, 1, 2])
def test_tiny_strided_maywrite(G, O, pc, hull_every):
    r = rng(7000 + hull_every)
    for trial in range(25):
        skels = _tiny_space(r, hull_every)
        run_parity(G, O, pc, skels, _tiny_records(r, 3000, len(skels), big=trial % 3 == 2))


@pytest.mark.parametrize("name", ["c3s", "c3h"])
def test_c3_brs_prefix_ragged(G, O, pc, name):
    c = R.config(name)
    run_parity(G, O, pc, c["skeletons"], R.gen_records(c, 0, 30_011))
    # every skeleton: records from each skeleton's range
    idx = np.concatenate([np.arange(k * c["n"] // 64, k * c["n"] // 64 + 300, dtype=np.uint64)
                          for k in range(64)])
    run_parity(G, O, pc, c["skeletons"], records_slice(c, idx), index_base=0)


def test_mixed_paths_one_space(G, O, pc):
    """Plan skeletons (C4 library), strided sweeps and hull skeletons in one
    design space, interleaved record by record so warps mix the paths."""
    c4 = R.config("c4")["skeletons"][:7]
    skels = c4 + R.config("c3s")["skeletons"][:4] + R.config("c3h")["skeletons"][:4]
    r = rng(31)
    n = 50_000
    sk = r.integers(0, len(skels), n)
    n0 = r.integers(256, 4096, n)
    one_d = np.isin(sk, [4, 5])
    rec = {"skx": ((sk << 16) | r.integers(0, 16, n)).astype(np.uint32),
           "nx": n0.astype(np.uint32),
           "ny": np.where(one_d, 1, np.where(sk == 6, 132, r.integers(256, 4096, n))).astype(np.uint32),
           "iters": r.integers(1, 1025, n).astype(np.uint32)}
    rec["nx"][sk == 6] = 2048
    run_parity(G, O, pc, skels, rec)


@pytest.mark.parametrize("name", ["c3s", "c3h"])
def test_c3_brs_full_size_sampled(G, O, pc, name):
    _full_size_check(G, O, pc, name, n_sample=8_000)


def test_hull_never_below_exact_on_gpu(G, O, pc):
    """The proven bound (N4h) on the device outputs: hull bytes >=
    exact bytes record by record (same skeletons, both modes)."""
    c = R.config("c3s")
    rec = R.gen_records(c, 0, 40_000)
    ex = G.Space(c["skeletons"], S.FX5600)
    hu = G.Space([dict(s, hull=True) for s in c["skeletons"]], S.FX5600)
    he, de, te = [x.cpu().numpy() for x in ex.eval(pc, G.Records.from_numpy(rec))]
    hh, dh, th = [x.cpu().numpy() for x in hu.eval(pc, G.Records.from_numpy(rec))]
    assert (hh.view(np.uint64) >= he.view(np.uint64)).all()
    assert (dh.view(np.uint64) >= de.view(np.uint64)).all()
    assert (hh != he).any()      # the workload does exercise the approximation
