"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bytes and the selected index must be bit-exact; times
are compared bitwise (the arithmetic is fixed-order IEEE binary64 on both
sides, DESIGN.md §3 N1), which is stricter than BASELINE.json's 1e-9
relative bound.

Sizes: every config at a size the oracle finishes in seconds (several tiles,
ragged tails), and C2/C3/C4 at their full BASELINE.json sizes in the launch
configuration bench.py uses, checked on sampled outputs plus size-independent
properties (argmin consistency, sharding invariance, generator identity).
"""
import math
import os

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import (assert_same, gpu_eval, oracle_problem, paper_pcie,
                               records_slice)
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


def run_parity(G, O, pc, skels, rec, gpu=S.FX5600, index_base=0):
    space = G.Space(skels, gpu)
    P = oracle_problem(O, skels, gpu)
    g = gpu_eval(G, space, pc, rec, index_base)
    o = P.eval(rec)
    assert_same(g, o)
    # best: GPU fused argmin == oracle argmin
    rc, b = space.best(pc, G.Records.from_numpy(rec), index_base=index_base)
    orc, ob = P.best(rec, index_base=index_base)
    assert b.index == ob.index
    if ob.index != G.UINT64_MAX:
        assert b.t_total_s == ob.t_total_s
        assert (b.h2d_bytes, b.d2h_bytes) == (ob.h2d_bytes, ob.d2h_bytes)
    assert (b.n_invalid, b.n_valid) == (ob.n_invalid, ob.n_valid)
    space.close()
    return g, o, b


def test_c1_full(G, O, pc):
    c = R.config("c1")
    rec = R.gen_records(c)
    g, o, b = run_parity(G, O, pc, c["skeletons"], rec)
    assert b.index == 5                      # oracle-pinned winner (App. B.1 reading)
    assert math.isinf(g[2][14])              # 512 threads x 20 regs: infeasible


def test_c2_full(G, O, pc):
    c = R.config("c2")
    run_parity(G, O, pc, c["skeletons"], R.gen_records(c))


def test_c3_prefix_ragged(G, O, pc):
    c = R.config("c3")
    run_parity(G, O, pc, c["skeletons"], R.gen_records(c, 0, 200_013), index_base=0)


def test_c4_prefix_every_skeleton(G, O, pc):
    c = R.config("c4")
    G_ = c["n"] // 16
    idx = np.concatenate([np.arange(-(-s * G_ // 16) * 16, -(-s * G_ // 16) * 16 + 4099)
                          for s in range(16)])
    rec = records_slice(c, idx)
    run_parity(G, O, pc, c["skeletons"], rec)


@pytest.mark.parametrize("n", [0, 1, 3, 5, 31, 33, 257, 4097])
def test_edge_lengths(G, O, pc, n):
    c = R.config("c2")
    rec = R.gen_records(c, 1000, 1000 + n)
    space = G.Space(c["skeletons"], S.FX5600)
    if n == 0:
        rc, b = space.best(pc, G.Records.from_numpy(rec))
        assert rc == G.ENOFEASIBLE and b.index == G.UINT64_MAX and b.n_valid == 0
        return
    run_parity(G, O, pc, c["skeletons"], rec, index_base=7)


def test_invalid_records(G, O, pc):
    c = R.config("c2")
    rec = R.gen_records(c, 0, 1000)
    rng_ = np.random.default_rng(3)
    bad = rng_.choice(1000, 100, replace=False)
    kinds = rng_.integers(0, 6, 100)
    for i, k in zip(bad, kinds):
        if k == 0:
            rec["skx"][i] = (3 << 16) | 1          # skeleton out of range
        elif k == 1:
            rec["skx"][i] = (rec["skx"][i] & 0xFFFF0000) | 16   # xform out of range
        elif k == 2:
            rec["nx"][i] = 0
        elif k == 3:
            rec["ny"][i] = (1 << 20) + 1
        elif k == 4:
            rec["iters"][i] = 0
        else:
            rec["nx"][i] = 0xFFFFFFFF
    space = G.Space(c["skeletons"], S.FX5600)
    space.invalid_count()
    g, o, b = run_parity(G, O, pc, c["skeletons"], rec)
    assert b.n_invalid == 100
    assert np.isnan(g[2][bad]).all() and (g[0][bad] == 0).all() and (g[1][bad] == 0).all()
    space2 = G.Space(c["skeletons"], S.FX5600)
    space2.eval(pc, G.Records.from_numpy(rec))
    assert space2.invalid_count() == 100
    assert space2.invalid_count() == 0
    rc, _ = space2.best(pc, G.Records.from_numpy(rec))
    assert rc == G.EBADCAND


def test_all_infeasible(G, O, pc):
    c = R.config("c1")
    rec = {"skx": np.full(100, 14, np.uint32), "nx": np.full(100, 64, np.uint32),
           "ny": np.full(100, 64, np.uint32), "iters": np.ones(100, np.uint32)}
    space = G.Space(c["skeletons"], S.FX5600)
    rc, b = space.best(pc, G.Records.from_numpy(rec))
    assert rc == G.ENOFEASIBLE and b.index == G.UINT64_MAX and b.n_valid == 100


def test_ties_lowest_global_index(G, O, pc):
    """HotSpot at 1024^2, 10 iterations: several transformations tie exactly;
    duplicated records tie by construction.  Lowest global index wins, also
    across tiles / CTAs."""
    sk = [S.s1_hotspot()]
    P = oracle_problem(O, sk)
    tt = [P.eval_one(x, 1024, 1024, 10)[3] for x in range(16)]
    best_x = min(range(16), key=lambda x: (tt[x], x))
    ties = [x for x in range(16) if tt[x] == tt[best_x]]
    n = 300_000
    r = np.random.default_rng(11)
    allowed = np.array([x for x in range(16) if tt[x] != tt[best_x]], np.uint32)
    skx = allowed[r.integers(0, allowed.size, n)]
    pos = sorted(int(p) for p in r.choice(n, 5, replace=False))
    for p in pos:
        skx[p] = ties[int(r.integers(0, len(ties)))]
    rec = {"skx": skx, "nx": np.full(n, 1024, np.uint32), "ny": np.full(n, 1024, np.uint32),
           "iters": np.full(n, 10, np.uint32)}
    space = G.Space(sk, S.FX5600)
    for base in (0, 5 * 10**8):
        rc, b = space.best(pc, G.Records.from_numpy(rec), index_base=base)
        assert b.index == base + pos[0] and b.t_total_s == tt[best_x]


def test_max_sizes(G, O, pc):
    c = R.config("c4")
    n = len(c["skeletons"])
    pts = [(1 << 20, 1 << 20), (1 << 20, 1), (1, 1 << 20), (1, 1), (2, 2), (3, 1 << 20)]
    rec = {k: [] for k in ("skx", "nx", "ny", "iters")}
    for s in range(n):
        for x in range(16):
            for (a, b_) in pts:
                rec["skx"].append((s << 16) | x)
                rec["nx"].append(a)
                rec["ny"].append(b_)
                rec["iters"].append(1 + (x * 37) % 1024)
    rec = {k: np.array(v, np.uint32) for k, v in rec.items()}
    run_parity(G, O, pc, c["skeletons"], rec)


def test_b200_like_gpu_model(G, O, pc):
    """Another GPU model (other occupancy / MWP regimes)."""
    c = R.config("c4")
    idx = np.arange(0, 10**9, 10**9 // 50_000)
    rec = records_slice(c, idx)
    run_parity(G, O, pc, c["skeletons"], rec, gpu=S.B200_LIKE)


def test_random_tiny_skeletons(G, O, pc):
    """Random tiny skeletons (empty / inverted / clamped boxes, R/W/RW, whole
    reads) with random per-transformation characteristics; many sizes each.
    Exercises the general cell sweep and the small-grid (non-saturated) model."""
    r = rng(2024)
    for trial in range(60):
        skels = []
        for _ in range(4):
            s, _, _ = random_tiny_skeleton(r, n_xforms=4)
            s["kx"] = [[{"tpb": int(r.choice([32, 64, 96, 128, 256, 512, 1024])),
                         "ipt": int(r.integers(1, 5)), "regs": int(r.integers(0, 40)),
                         "smem": int(r.choice([0, 0, 512, 4096, 20000])),
                         "total": float(r.integers(20, 200)), "coal": float(r.integers(0, 12)),
                         "uncoal": float(r.choice([0, 0, 3, 10])), "upm": 32.0,
                         "lbpw": float(r.choice([64, 128])), "synch": float(r.integers(0, 3))}
                        for _ in s["kernels"]] for _ in range(4)]
            for row in s["kx"]:
                for c_ in row:
                    c_["total"] = max(c_["total"], c_["coal"] + c_["uncoal"])
            skels.append(s)
        n = 2048
        rec = {"skx": ((r.integers(0, 4, n) << 16) | r.integers(0, 4, n)).astype(np.uint32),
               "nx": r.integers(1, 40, n).astype(np.uint32),
               "ny": r.integers(1, 40, n).astype(np.uint32),
               "iters": r.integers(1, 50, n).astype(np.uint32)}
        gpu = S.FX5600 if trial % 2 == 0 else S.B200_LIKE
        run_parity(G, O, pc, skels, rec, gpu=gpu)


def test_random_multikernel_all_sizes(G, O, pc):
    skels = S.random_skeletons(0xC0FFEE, 24)
    r = rng(99)
    n = 60_000
    small = r.random(n) < 0.3
    nx = np.where(small, r.integers(1, 300, n), r.integers(256, 1 << 20, n))
    ny = np.where(small, r.integers(1, 300, n), r.integers(1, 1 << 14, n))
    rec = {"skx": ((r.integers(0, 24, n) << 16) | r.integers(0, 16, n)).astype(np.uint32),
           "nx": nx.astype(np.uint32), "ny": ny.astype(np.uint32),
           "iters": r.integers(1, 1025, n).astype(np.uint32)}
    run_parity(G, O, pc, skels, rec)
    run_parity(G, O, pc, skels, rec, gpu=S.B200_LIKE)


def test_device_generator_matches_numpy(G):
    for name in ("c2", "c3", "c4"):
        c = R.config(name)
        for start, count in ((0, 5000), (c["n"] - 4099, 4099), (c["n"] // 3 + 7, 12345)):
            d = G.synth_records(c, start, count)
            torch.cuda.synchronize()
            h = R.gen_records(c, start, start + count)
            for k, t in zip(("skx", "nx", "ny", "iters"), (d.skx, d.nx, d.ny, d.iters)):
                assert np.array_equal(t.cpu().numpy().view(np.uint32), h[k]), (name, k)


def test_best_host_and_async_and_combine(G, O, pc):
    c = R.with_n(R.config("c3"), 3_000_000)
    space = G.Space(c["skeletons"], S.FX5600)
    dev = G.synth_records(c)
    rc, b = space.best(pc, dev)
    # e2e host path (pinned records, chunked copies) gives the same answer
    host = {k: torch.from_numpy(v.view(np.int32)).pin_memory()
            for k, v in R.gen_records(c).items()}
    rc2, b2 = space.best_host(pc, host)
    assert b2.as_tuple() == b.as_tuple()
    # shards accumulated in one device slot == whole batch
    out = G.best_result_tensor()
    bounds = [0, 1, 999_999, 1_000_000, 2_345_678, c["n"]]
    for i in range(len(bounds) - 1):
        bt = dev.batch(index_base=bounds[i], start=bounds[i], stop=bounds[i + 1])
        if i == 0:
            out.copy_(torch.tensor([0, -1, 0, 0, 0, 0], dtype=torch.int64))
            out[0:1].view(torch.float64).fill_(math.inf)
        space.best_async(pc, bt, out, accumulate=True)
    torch.cuda.synchronize()
    assert G.result_from_tensor(out).as_tuple() == b.as_tuple()
    # per-shard results -> device combine == host combine == whole
    parts = G.best_result_tensor(5)
    res = []
    for i in range(5):
        bt = dev.batch(index_base=bounds[i], start=bounds[i], stop=bounds[i + 1])
        space.best_async(pc, bt, parts[6 * i:6 * i + 6], accumulate=False)
    torch.cuda.synchronize()
    res = [G.result_from_tensor(parts, i) for i in range(5)]
    comb = G.best_result_tensor()
    G.best_combine(parts, 5, comb)
    torch.cuda.synchronize()
    assert G.result_from_tensor(comb).as_tuple() == b.as_tuple()
    assert G.best_combine_host(res).as_tuple() == b.as_tuple()
    # oracle agrees on the winner's record
    P = oracle_problem(O, c["skeletons"])
    one = R.gen_records(c, b.index, b.index + 1)
    ok, h, d, t = P.eval_one(int(one["skx"][0]), int(one["nx"][0]), int(one["ny"][0]),
                             int(one["iters"][0]))
    assert (h, d, t) == (b.h2d_bytes, b.d2h_bytes, b.t_total_s)


def _full_size_check(G, O, pc, name, n_sample=20_000, chunk=1 << 24):
    """Full BASELINE.json size, bench launch configuration (device-generated
    records, one fused best launch over all of them)."""
    c = R.config(name)
    N = c["n"]
    space = G.Space(c["skeletons"], S.FX5600)
    dev = G.synth_records(c)
    rc, b = space.best(pc, dev)
    assert rc == G.OK and b.n_valid == N
    P = oracle_problem(O, c["skeletons"])
    # sampled outputs: eval chunks on the GPU vs the oracle one by one
    r = rng(sum(map(ord, name)))
    idx = np.unique(np.concatenate([r.integers(0, N, n_sample), [0, N - 1, b.index]]))
    gh = np.empty(idx.size, np.uint64)
    gd = np.empty(idx.size, np.uint64)
    gt = np.empty(idx.size, np.float64)
    eh = torch.empty(chunk, dtype=torch.int64, device="cuda")
    ed = torch.empty(chunk, dtype=torch.int64, device="cuda")
    et = torch.empty(chunk, dtype=torch.float64, device="cuda")
    gmin = (math.inf, None)
    for s in range(0, N, chunk):
        e = min(N, s + chunk)
        sel = (idx >= s) & (idx < e)
        if not sel.any():
            continue
        sub = G.Records(dev.skx[s:e], dev.nx[s:e], dev.ny[s:e], dev.iters[s:e])
        space.eval(pc, sub, index_base=s, out=(eh[:e - s], ed[:e - s], et[:e - s]))
        torch.cuda.synchronize()
        loc = torch.from_numpy(idx[sel] - s).cuda()
        gh[sel] = eh[loc].cpu().numpy().view(np.uint64)
        gd[sel] = ed[loc].cpu().numpy().view(np.uint64)
        gt[sel] = et[loc].cpu().numpy()
    rec = records_slice(c, idx)
    o = P.eval(rec)
    assert_same((gh, gd, gt), o)
    # the fused argmin is consistent with the sampled outputs and the oracle
    k = int(np.nonzero(idx == b.index)[0][0])
    assert gt[k] == b.t_total_s and gh[k] == b.h2d_bytes and gd[k] == b.d2h_bytes
    finite = np.isfinite(gt)
    assert b.t_total_s <= gt[finite].min()
    # sharding invariance over 8 shards (the multi-GPU partition)
    res = []
    for rnk in range(8):
        lo, hi = N * rnk // 8, N * (rnk + 1) // 8
        res.append(space.best(pc, dev, batch=dev.batch(index_base=lo, start=lo, stop=hi))[1])
    assert G.best_combine_host(res).as_tuple() == b.as_tuple()
    space.close()
    return b


def test_c2_full_size_sampled(G, O, pc):
    _full_size_check(G, O, pc, "c2")


def test_c3_full_size_sampled(G, O, pc):
    # the full-size argmin and checksums against the oracle: test_gpu_golden.py
    _full_size_check(G, O, pc, "c3")


def test_c4_full_size_sampled(G, O, pc):
    _full_size_check(G, O, pc, "c4", n_sample=30_000)


def test_random_tiny_skeletons_large_sizes(G, O, pc):
    """Tiny random skeletons at log-uniform sizes up to 2^20: keys inside and
    outside each skeleton's compiled usage-plan domain, in the same warps."""
    r = rng(4242)
    for trial in range(20):
        skels = [random_tiny_skeleton(r, n_xforms=2)[0] for _ in range(6)]
        n = 4096
        rec = {"skx": ((r.integers(0, 6, n) << 16) | r.integers(0, 2, n)).astype(np.uint32),
               "nx": np.exp2(r.uniform(0, 20, n)).astype(np.uint32),
               "ny": np.exp2(r.uniform(0, 20, n)).astype(np.uint32),
               "iters": r.integers(1, 50, n).astype(np.uint32)}
        run_parity(G, O, pc, skels, rec)
