"""Multi-process (gloo, world_size 2-4) tests of the multi-GPU host logic:
contiguous sharding with global index_base, and the min-loc combine after an
all-gather (the same grophecy_best_combine_host the GPU path mirrors with its
combine kernel).  Shard bests come from the oracle (test infrastructure); the
product supplies the sharding, the collective glue and the combine."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from synth import records as R
from synth import skeletons as S


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, case, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import oracle as O
        from paper_conf_ipps_boyermk13_b200 import dist as D
        from paper_conf_ipps_boyermk13_b200 import grophecy as G
        skels, rec, n = case[:3]
        lo, hi = D.shard_range(n, rank, world)
        rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
        P = O.Problem(skels, S.FX5600, link)
        part = {k: v[lo:hi] for k, v in rec.items()}
        if len(case) > 3 and case[3] == "groups":
            groups = _oracle_groups(G, P, part, lo)
            keys = [D.record_key(*[part[f][i] for f in ("skx", "nx", "ny", "iters")])
                    for i in ((0, hi - lo - 1) if hi > lo else ())]
            fixed = D.fix_shard_groups(groups, hi - lo, keys[0] if keys else None,
                                       keys[-1] if keys else None)
            q.put((rank, [_gtuple(g) for g in fixed]))
            return
        _, ob = P.best(part, index_base=lo, nthreads=1)
        local = G.BestResult(ob.t_total_s, ob.index, ob.h2d_bytes, ob.d2h_bytes, ob.n_invalid,
                             ob.n_valid)
        out = D.minloc_host(local)
        q.put((rank, out.as_tuple()))
    finally:
        dist.destroy_process_group()


def _oracle_groups(G, P, rec, base):
    """Per-shard groups from the oracle as GroupResult (bytes left 0)."""
    f, cnt, bi, bt = P.group_best(rec, index_base=base)
    return [G.GroupResult(float(bt[g]), int(f[g]), int(cnt[g]), int(bi[g]), 0, 0)
            for g in range(len(f))]


def _gtuple(g):
    return (g.first, g.count, g.best_index, float(np.float64(g.best_t_s).view(np.uint64)))


def _run(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return dict(res)


def _oracle_best(O, case):
    skels, rec, n = case
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    P = O.Problem(skels, S.FX5600, link)
    _, b = P.best(rec)
    return (b.t_total_s, b.index, b.h2d_bytes, b.d2h_bytes, b.n_invalid, b.n_valid)


def test_shard_range_partitions():
    from paper_conf_ipps_boyermk13_b200.dist import shard_range
    for n in (0, 1, 7, 16, 10**6, 10**9, 10**9 + 3):
        for world in (1, 2, 3, 4, 8):
            prev = 0
            for r in range(world):
                lo, hi = shard_range(n, r, world)
                assert lo == prev and hi >= lo
                assert abs((hi - lo) - n / world) < 1
                prev = hi
            assert prev == n


@pytest.mark.parametrize("world", [2, 4])
def test_minloc_over_gloo_equals_global_best(O, world):
    c = R.with_n(R.config("c2"), 6000)
    rec = R.gen_records(c)
    case = (c["skeletons"], rec, c["n"])
    res = _run(world, case)
    want = _oracle_best(O, case)
    for r in range(world):
        assert res[r] == want


def test_minloc_tie_across_shard_boundary(O):
    """Equal best times on both sides of the shard boundary: the lower global
    index (rank 0's) must win on every rank."""
    sk = [S.s1_hotspot()]
    n = 64
    rec = {"skx": np.full(n, 7, np.uint32), "nx": np.full(n, 1024, np.uint32),
           "ny": np.full(n, 1024, np.uint32), "iters": np.full(n, 10, np.uint32)}
    rec["skx"][31] = 0      # x = 0 ties with x = 8 and 12 (exactly equal totals)
    rec["skx"][32] = 8
    rec["skx"][40] = 12
    case = (sk, rec, n)
    want = _oracle_best(O, case)
    res = _run(2, case)
    assert want[1] in (31, 32, 40)
    assert res[0] == res[1] == want


def test_minloc_invalid_and_empty_shards(O):
    c = R.config("c1")
    rec = R.gen_records(c)
    rec["nx"][:8] = 0          # rank 0's shard entirely invalid
    case = (c["skeletons"], rec, c["n"])
    res = _run(2, case)
    want = _oracle_best(O, case)
    assert res[0] == res[1] == want and want[4] == 8


def _group_case(n, seed, n_xf=16):
    """Records with runs of 1..n/3 equal keys (some spanning several shards),
    invalid runs and transformations out of order."""
    rng = np.random.default_rng(seed)
    skx, nx, ny, it = [], [], [], []
    while len(skx) < n:
        run = int(rng.integers(1, max(2, n // 3)))
        s_, x_, y_, i_ = int(rng.integers(0, 3)), int(rng.integers(256, 4096)), 0, int(rng.integers(1, 50))
        y_ = x_
        if rng.random() < 0.1:
            x_ = 0          # invalid run
        for _ in range(run):
            skx.append((s_ << 16) | int(rng.integers(0, n_xf)))
            nx.append(x_)
            ny.append(y_)
            it.append(i_)
    rec = {"skx": np.array(skx[:n], np.uint32), "nx": np.array(nx[:n], np.uint32),
           "ny": np.array(ny[:n], np.uint32), "iters": np.array(it[:n], np.uint32)}
    return rec


def _full_groups(O, skels, rec):
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    P = O.Problem(skels, S.FX5600, link)
    f, cnt, bi, bt = P.group_best(rec)
    return [(int(f[g]), int(cnt[g]), int(bi[g]), float(np.float64(bt[g]).view(np.uint64)))
            for g in range(len(f))]


def test_shard_group_fixups_pure(O):
    """Every split of a record set into 1..6 contiguous shards: per-shard
    groups + fix-up == the groups of the whole set (NEXT-1 cross-shard)."""
    from paper_conf_ipps_boyermk13_b200 import dist as D
    from paper_conf_ipps_boyermk13_b200 import grophecy as G
    skels = R.config("c2")["skeletons"]
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    P = O.Problem(skels, S.FX5600, link)
    for seed in range(12):
        n = 40 + 7 * seed
        rec = _group_case(n, seed)
        want = _full_groups(O, skels, rec)
        rng = np.random.default_rng(100 + seed)
        for world in (1, 2, 3, 4, 6):
            cuts = sorted(rng.integers(0, n + 1, world - 1).tolist())   # empty shards allowed
            bounds = [0] + cuts + [n]
            infos, locals_ = [], []
            for r in range(world):
                lo, hi = bounds[r], bounds[r + 1]
                part = {k: v[lo:hi] for k, v in rec.items()}
                gs = _oracle_groups(G, P, part, lo) if hi > lo else []
                keys = [D.record_key(*[part[f][i] for f in ("skx", "nx", "ny", "iters")])
                        for i in ((0, hi - lo - 1) if hi > lo else ())]
                infos.append((hi - lo, keys[0] if keys else None, keys[-1] if keys else None,
                              gs[0] if gs else None, gs[-1] if gs else None, len(gs)))
                locals_.append(gs)
            fix = D.shard_group_fixups(infos)
            got = []
            for r in range(world):
                got += [_gtuple(g) for g in D.apply_group_fixup(locals_[r], fix[r])]
            assert got == want, (seed, world, bounds)


@pytest.mark.parametrize("world", [2, 4])
def test_group_fixup_over_gloo(O, world):
    skels = R.config("c2")["skeletons"]
    rec = _group_case(45, 7)
    want = _full_groups(O, skels, rec)
    res = _run(world, (skels, rec, 45, "groups"))
    got = []
    for r in range(world):
        got += res[r]
    assert got == want


@pytest.mark.parametrize("n,world,stripes", [(10**9, 8, 16), (10**9, 2, 16), (1000, 4, 16),
                                             (10**6, 3, 5), (0, 2, 4)])
def test_striped_chunks_partition(n, world, stripes):
    """bench.py's N > 1 shards: every record exactly once, tile-aligned
    chunk starts, every rank's chunks in increasing order."""
    from paper_conf_ipps_boyermk13_b200 import dist as D
    chunks = []
    for r in range(world):
        mine = [c for c in D.striped_chunks(n, r, world, stripes) if c[1] > c[0]]
        assert all(a < b for a, b in mine)
        assert all(mine[i][1] <= mine[i + 1][0] for i in range(len(mine) - 1))
        assert all(a % 512 == 0 for a, _ in mine)
        chunks += mine
    pos = 0
    for a, b in sorted(chunks):
        assert a == pos
        pos = b
    assert pos == n


@pytest.mark.parametrize("n,world,stripes", [(10**9, 8, 16), (10**9, 2, 16), (10**7, 3, 5),
                                             (5000, 4, 16), (0, 2, 4), (123457, 7, 3)])
def test_stripe_layout_partition(n, world, stripes):
    """dist.stripe_layout: the ranks' stripe batches + tails cover [0, n)
    exactly once, and the local -> global map of the stripe batch is the one
    grophecy_batch documents (increasing, so ties stay lowest-index)."""
    import numpy as np
    from paper_conf_ipps_boyermk13_b200 import dist as D
    total = 0
    pieces = []
    for r in range(world):
        L, n_main, (t_lo, t_hi) = D.stripe_layout(n, r, world, stripes)
        assert L % 4096 == 0 and n_main == (stripes * L)
        total += n_main + t_hi - t_lo
        for k in range(stripes if L else 0):
            g0 = D.stripe_global_index(k * L, r, world, L)
            assert g0 == (r + world * k) * L
            pieces.append((g0, g0 + L))
        if t_hi > t_lo:
            pieces.append((t_lo, t_hi))
        if L:
            i = np.array([0, L - 1, L, n_main - 1])
            g = [D.stripe_global_index(int(v), r, world, L) for v in i]
            assert g == sorted(g)
    assert total == n
    pieces.sort()
    pos = 0
    for a, b in pieces:
        assert a == pos
        pos = b
    assert pos == n
