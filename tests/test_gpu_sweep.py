"""The sweep path's layout cases: design points of 16 records
in any fixed transformation order, the batch's last partial tile, mixed
orders (the tile falls back to the general path), all against the oracle.
Best and eval are compared record by record / by argmin; index_base and
ragged sizes exercised."""
import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import assert_same, gpu_eval, oracle_problem, paper_pcie

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


def check(G, O, skels, rec, index_base=0):
    pc = paper_pcie(G)
    space = G.Space(skels, S.FX5600)
    P = oracle_problem(O, skels)
    assert_same(gpu_eval(G, space, pc, rec, index_base), P.eval(rec))
    rc, b = space.best(pc, G.Records.from_numpy(rec), index_base=index_base)
    orc, ob = P.best(rec, index_base=index_base)
    assert (b.index, b.n_valid, b.n_invalid) == (ob.index, ob.n_valid, ob.n_invalid)
    assert b.t_total_s == ob.t_total_s and (b.h2d_bytes, b.d2h_bytes) == (ob.h2d_bytes, ob.d2h_bytes)
    space.close()


def permuted(rec, perm):
    """Reorder the 16 records of every design point by `perm` (positions)."""
    n = len(rec["skx"])
    idx = (np.arange(n) // 16) * 16 + np.asarray(perm)[np.arange(n) % 16]
    return {k: v[idx] for k, v in rec.items()}


@pytest.mark.parametrize("order", ["reversed", "random", "repeat"])
def test_fixed_transformation_order(G, O, order):
    c = R.config("c4")
    n = 3 * 4096 + 16 * 37            # three full CTA tiles and a partial one
    base = 16 * 1000
    rec = R.gen_records(c, base, base + n)
    rng = np.random.default_rng(17)
    perm = {"reversed": np.arange(16)[::-1], "random": rng.permutation(16),
            "repeat": np.array([0, 3, 3, 1, 15, 2, 7, 7, 4, 5, 6, 8, 9, 10, 11, 12])}[order]
    check(G, O, c["skeletons"], permuted(rec, perm), index_base=base)


def test_mixed_orders_fall_back(G, O):
    """One design point in a different order: its CTA tile is not a sweep
    tile (general path); the others still are."""
    c = R.config("c4")
    n = 4 * 4096
    rec = R.gen_records(c, 0, n)
    rec = permuted(rec, np.arange(16)[::-1])
    i = 4096 + 16 * 5                  # one design point of tile 1 in natural order
    for k in rec:
        rec[k][i:i + 16] = rec[k][i:i + 16][::-1]
    check(G, O, c["skeletons"], rec)


@pytest.mark.parametrize("n", [4096 + 16, 8192 - 16, 4096 * 5 + 16 * 255, 4096 * 2 + 7])
def test_partial_last_tile(G, O, n):
    c = R.config("c4")
    start = 16 * 62_500_000 // 16     # inside the skeleton-major ranges
    rec = R.gen_records(c, start, start + n)
    check(G, O, c["skeletons"], rec, index_base=start)


def test_large_counts_u64_usage(G, O):
    """Sweep tiles whose byte counts exceed 2^32 (random multi-kernel
    skeletons at nx, ny around 2^15, 8-byte elements: counts up to 2^33, work
    counts still below the fast path's 2^30): the usage takes the 64-bit
    evaluation (the 32-bit one only when a per-skeleton bound proves every
    count < 2^32); a tile mixing both kinds of sizes, against the oracle."""
    c = R.config("c3")
    n = 2 * 4096
    rec = R.gen_records(c, 0, n)
    rng = np.random.default_rng(99)
    g = n // 16
    big = rng.integers(30000, 32768, g).astype(np.uint32)
    small = rng.integers(256, 2048, g).astype(np.uint32)
    pick = rng.random(g) < 0.7
    nx = np.where(pick, big, small)
    ny = np.where(pick, big[::-1], small[::-1])
    rec["nx"] = np.repeat(nx, 16)
    rec["ny"] = np.repeat(ny, 16)
    check(G, O, c["skeletons"], rec)


def fewer_xforms(cfg, X):
    """The config with every skeleton cut to its first X transformations
    (design points of X records: the sweep's design-point size follows the
    space)."""
    c = dict(cfg)
    c["skeletons"] = [dict(s, kx=s["kx"][:X]) for s in cfg["skeletons"]]
    c["n_xforms"] = X
    return c


@pytest.mark.parametrize("X", [8, 4])
def test_design_points_of_fewer_transformations(G, O, X):
    """Spaces whose skeletons have 8 or 4 transformations run the sweep with
    design points of that size: several full CTA tiles, a partial last one,
    a reversed order (still a sweep), an index base inside the workload."""
    c = fewer_xforms(R.config("c4"), X)
    swt = 256 * X
    n = 5 * swt + X * 37
    base = X * 1_000_003
    rec = R.gen_records(c, base, base + n)
    check(G, O, c["skeletons"], rec, index_base=base)
    rev = {k: v.reshape(-1, X)[:, ::-1].reshape(-1).copy() for k, v in rec.items()}
    check(G, O, c["skeletons"], rev, index_base=base)


@pytest.mark.parametrize("X", [8, 4])
def test_fewer_transformations_bench_layout(G, O, X):
    """C2-shaped spaces (three skeletons, skeleton boundaries inside CTA
    tiles) with X transformations: eval record by record and the argmin vs
    the oracle; the ragged batch end (not a whole design point) goes to the
    general path."""
    c = fewer_xforms(R.config("c2"), X)
    n = 200_003
    rec = R.gen_records(c, 0, n)
    check(G, O, c["skeletons"], rec)


@pytest.mark.parametrize("two", ["0", "1"])
@pytest.mark.parametrize("grid", [1, 3])
def test_many_tiles_per_cta(G, O, monkeypatch, grid, two):
    """A sweep grid of 1 or 3 CTAs (GROPHECY_SWEEP_GRID): every CTA runs
    dozens of tiles back to back through its per-tile barriers and counters,
    with the skeleton (the staged usage table) changing every 4 tiles,
    non-uniform tiles (one design point in another order) between uniform
    ones, and a partial last tile; eval and the argmin vs the oracle."""
    c = R.config("c4")
    c = dict(c, n=16 * 4 * 4096)       # 16 skeletons, a boundary every 4 tiles
    n = c["n"] - 16 * 29               # partial last tile
    rec = R.gen_records(c, 0, n)
    for t in (5, 6, 17, 40):           # tiles with one design point reversed
        i = t * 4096 + 16 * 7
        for k in rec:
            rec[k][i:i + 16] = rec[k][i:i + 16][::-1]
    monkeypatch.setenv("GROPHECY_SWEEP_GRID", str(grid))
    monkeypatch.setenv("GROPHECY_SWEEP_TWO", two)   # one- and two-skeleton tiles
    check(G, O, c["skeletons"], rec)


def test_interleaved_design_points_general_path(G, O):
    """The records of design point pairs interleaved record by record (equal
    keys not adjacent): no sweep tile; the general path groups the equal keys
    of each 32 records (one usage evaluation per key); vs the oracle."""
    c = R.config("c4")
    n = 6 * 4096 + 32 * 11 + 5
    base = 16 * 3_000_000
    rec = R.gen_records(c, base, base + n)
    i = np.arange(n)
    blk = (i // 32) * 32
    idx = np.where(blk + 32 <= n, blk + (i % 2) * 16 + (i % 32) // 2, i)
    check(G, O, c["skeletons"], {k: v[idx] for k, v in rec.items()}, index_base=base)


@pytest.mark.parametrize("two", ["0", "1"])
@pytest.mark.parametrize("name", ["c2", "c3"])
def test_skeleton_boundaries_inside_tiles(G, O, monkeypatch, name, two):
    """Skeleton boundaries inside CTA tiles and inside warp tiles (C2 / C3
    prefixes re-cut so that every few tiles hold two skeletons, one tile three),
    with two-skeleton sweep tiles on and off (GROPHECY_SWEEP_TWO); vs the oracle."""
    c = R.config(name)
    k = len(c["skeletons"])
    # records of consecutive skeleton ranges, cut at design points 4096*t + 16*(37 + 11 t)
    parts, start = [], 0
    for t in range(min(k, 6)):
        lo = (t * c["n"] // k) // 16 * 16
        n_t = 4096 + 16 * (37 + 11 * t) if t != 3 else 16 * 5   # (a 5-design-point run: 3 skeletons in a tile)
        parts.append(R.gen_records(c, lo, lo + n_t))
    rec = {f: np.concatenate([p[f] for p in parts]) for f in parts[0]}
    monkeypatch.setenv("GROPHECY_SWEEP_TWO", two)
    check(G, O, c["skeletons"], rec)
