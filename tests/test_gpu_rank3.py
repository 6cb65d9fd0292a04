"""GPU parity for rank-3 arrays (N4r): random
tiny rank-3 skeletons — dense and strided sections, may-writes, the hull
mode, plane ranges that depend on the size — through the C ABI against the
oracle, bitwise, at small and large sizes, mixed with 2-D skeletons in the
same batches (general device path: rank-3 skeletons have no usage plan)."""
import numpy as np
import pytest

from tests.gpu_helpers import paper_pcie
from tests.test_gpu_parity import run_parity
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


def _records(r, n, n_sk, big=False):
    if big:
        nx = np.exp2(r.uniform(0, 14, n)).astype(np.uint32)
        ny = np.exp2(r.uniform(0, 14, n)).astype(np.uint32)
    else:
        nx = r.integers(1, 40, n).astype(np.uint32)
        ny = r.integers(1, 40, n).astype(np.uint32)
    return {"skx": ((r.integers(0, n_sk, n) << 16) | r.integers(0, 2, n)).astype(np.uint32),
            "nx": nx, "ny": ny, "iters": r.integers(1, 50, n).astype(np.uint32)}


@pytest.mark.parametrize("mode", ["dense", "strided", "hull"])
def test_tiny_rank3(G, O, pc, mode):
    r = rng({"dense": 9500, "strided": 9600, "hull": 9700}[mode])
    for trial in range(20):
        skels = []
        for i in range(6):
            s, _, _ = random_tiny_skeleton(r, n_xforms=2, strided=mode == "strided",
                                           maywrite=True, hull=mode == "hull" and i % 2 == 0,
                                           rank3=i != 5)      # one 2-D skeleton in the space
            skels.append(s)
        run_parity(G, O, pc, skels, _records(r, 2000, len(skels), big=trial % 3 == 2))


def test_stencil_3d(G, O, pc):
    """A 3-D 7-point stencil sweep, planes = ny/8 (size-dependent), two
    ping-pong arrays: in [P][R][C] read, out interior written, then swapped."""
    from tests.tiny import DUMMY_KX

    def arr():
        return {"name": "a", "rows": (0, 0, 8, 0), "cols": (0, 8, 0, 0), "planes": (0, 0, 1, 0),
                "elem_bytes": 4, "liveout": True}

    def reg(k, a, mode, inner):
        lo = (1, 0, 0, 0) if inner else (0, 0, 0, 0)
        return {"kernel": k, "array": a, "mode": mode, "whole": False,
                "p0": lo, "p1": (-1, 0, 1, 0) if inner else (0, 0, 1, 0),
                "r0": lo, "r1": (-1, 0, 8, 0) if inner else (0, 0, 8, 0),
                "c0": lo, "c1": (-1, 8, 0, 0) if inner else (0, 8, 0, 0)}

    sk = {"name": "stencil3d", "arrays": [arr(), arr()],
          "kernels": [{"name": "k0", "work": (0, 0, 0, 8), "per_iter": True},
                      {"name": "k1", "work": (0, 0, 0, 8), "per_iter": True}],
          "regions": [reg(0, 0, "R", False), reg(0, 1, "W", True),
                      reg(1, 1, "R", False), reg(1, 0, "W", True)],
          "kx": [[DUMMY_KX] * 2] * 2}
    r = rng(9800)
    n = 4096
    rec = {"skx": r.integers(0, 2, n).astype(np.uint32),
           "nx": r.integers(1, 300, n).astype(np.uint32),
           "ny": r.integers(1, 300, n).astype(np.uint32),
           "iters": r.integers(1, 20, n).astype(np.uint32)}
    run_parity(G, O, pc, [sk], rec)
