"""GPU parity for the NEXT rows: time components (grophecy_eval_parts) and
best transformation per group (grophecy_group_best) against the oracle."""
import math

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import oracle_problem, paper_pcie, records_slice

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


def _bits(x):
    return np.asarray(x, np.float64).view(np.uint64)


def test_eval_parts_parity(G, O):
    c = R.config("c4")
    idx = np.arange(0, 10**9, 10**9 // 40_000, dtype=np.uint64)
    rec = records_slice(c, idx)
    rec["nx"][:50] = 0   # some invalid records
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    out = space.eval_parts(pc, G.Records.from_numpy(rec))
    torch.cuda.synchronize()
    h, d, t, ti, to, th, td = [o.cpu().numpy() for o in out]
    P = oracle_problem(O, c["skeletons"])
    for k in range(0, len(idx), 7):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, parts = P.eval_parts_one(*a)
        got = (ti[k], to[k], th[k], td[k])
        if not ok:
            assert all(math.isnan(v) for v in got) and math.isnan(t[k])
        else:
            assert _bits(got).tolist() == _bits(parts).tolist(), (k, a)
            assert t[k] == ((to[k] + a[3] * ti[k]) + th[k]) + td[k]


def _check_groups(G, O, skels, rec, base=0, cap=None):
    space = G.Space(skels, S.FX5600)
    pc = paper_pcie(G)
    rc, ng, res = space.group_best(pc, G.Records.from_numpy(rec), index_base=base, capacity=cap)
    P = oracle_problem(O, skels)
    f, cnt, bi, bt = P.group_best(rec, index_base=base)
    assert ng == len(f)
    for g, r in enumerate(res):
        assert (r.first, r.count, r.best_index) == (int(f[g]), int(cnt[g]), int(bi[g]))
        assert _bits([r.best_t_s]) == _bits([bt[g]])
        if r.best_index != G.UINT64_MAX:
            ok, h, d, t = P.eval_one(*[int(rec[k][r.best_index - base])
                                       for k in ("skx", "nx", "ny", "iters")])
            assert (h, d) == (r.h2d_bytes, r.d2h_bytes)
    return rc, ng, res


def test_group_best_c1_c2(G, O):
    c = R.config("c1")
    rc, ng, res = _check_groups(G, O, c["skeletons"], R.gen_records(c))
    assert ng == 1 and res[0].best_index == 5
    c = R.config("c2")
    _check_groups(G, O, c["skeletons"], R.gen_records(c, 0, 100_003), base=5)


def test_group_best_irregular_runs(G, O):
    """Runs of 1..3000 records (crossing 1024-record blocks), invalid and
    infeasible records inside groups, groups with no feasible candidate."""
    c = R.config("c4")
    rng = np.random.default_rng(21)
    rec = {k: [] for k in ("skx", "nx", "ny", "iters")}
    while len(rec["skx"]) < 40_000:
        s = int(rng.integers(0, 16))
        L = int(rng.choice([1, 2, 16, 17, 100, 1500, 3000]))
        n0 = int(rng.integers(256, 8192))
        it = int(rng.integers(1, 1025))
        allbad = rng.random() < 0.05
        for _ in range(L):
            x = int(rng.integers(0, 16))
            if allbad:
                x = 16          # invalid transformation
            elif rng.random() < 0.02:
                x = 17
            rec["skx"].append((s << 16) | x)
            rec["nx"].append(n0)
            rec["ny"].append(n0 if s not in (4, 5) else 1)
            rec["iters"].append(it)
    rec = {k: np.array(v, np.uint32) for k, v in rec.items()}
    _check_groups(G, O, c["skeletons"], rec, base=123)


def test_group_best_capacity(G, O):
    c = R.config("c2")
    rec = R.gen_records(c, 0, 1600)   # 100 groups of 16
    rc, ng, res = _check_groups(G, O, c["skeletons"], rec, cap=40)
    assert rc == G.ELIMIT and ng == 100 and len(res) == 40


def test_crossover_parity(G, O):
    """grophecy_crossover on eval_parts outputs vs oracle_crossover: per-
    candidate and scalar CPU iteration times, invalid records (NaN), never-
    winning candidates (c <= t_iter)."""
    c = R.config("c4")
    idx = np.arange(0, 10**9, 10**9 // 20_000, dtype=np.uint64)
    rec = records_slice(c, idx)
    rec["nx"][:20] = 0
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    h, d, t, ti, to, th, td = space.eval_parts(pc, G.Records.from_numpy(rec))
    rng = np.random.default_rng(3)
    # CPU time per iteration: 0.1x .. 10x of the GPU's per-iteration time
    scale = torch.from_numpy(10.0 ** rng.uniform(-1, 1, len(idx))).cuda()
    cpu = torch.where(torch.isfinite(ti) & (ti > 0), ti * scale, torch.full_like(ti, 1e-3))
    for arg in (cpu, 2.5e-4):
        nbe, imin = G.crossover(ti, to, th, td, arg)
        torch.cuda.synchronize()
        nb = nbe.cpu().numpy()
        im = imin.cpu().numpy().view(np.uint64)
        a = [x.cpu().numpy() for x in (ti, to, th, td)]
        cc = cpu.cpu().numpy() if not isinstance(arg, float) else np.full(len(idx), arg)
        for k in range(len(idx)):
            v, m = O.crossover(a[0][k], a[1][k], a[2][k], a[3][k], cc[k])
            assert (math.isnan(v) and math.isnan(nb[k])) or _bits([v]) == _bits([nb[k]]), k
            assert m == int(im[k]), (k, v, m, im[k])
        assert np.isinf(nb).any() and np.isfinite(nb).any()


def test_group_speedup_parity(G, O):
    c = R.config("c2")
    rec = R.gen_records(c, 0, 16 * 500)
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    rc, ng, gt = space.group_best(pc, G.Records.from_numpy(rec), as_tensor=True)
    assert ng == 500
    rng = np.random.default_rng(9)
    tcpu = torch.from_numpy(rng.uniform(1e-3, 10.0, ng)).cuda()
    sp = G.group_speedup(gt[:6 * ng], tcpu).cpu().numpy()
    best_t = gt[:6 * ng].view(ng, 6)[:, 0].cpu().numpy().view(np.float64)
    tc = tcpu.cpu().numpy()
    for g in range(ng):
        assert _bits([sp[g]]) == _bits([O.speedup(tc[g], best_t[g])])


def test_group_best_sharded_fixup(G, O):
    """Shards of a record set on one GPU (as the ranks would hold them), the
    pure cross-shard fix-up, and the whole set's groups (GPU and oracle)."""
    from paper_conf_ipps_boyermk13_b200 import dist as D
    c = R.config("c2")
    rec = R.gen_records(c, 0, 16 * 300)
    # irregular group lengths: drop random records so runs are 5..16 long
    rng = np.random.default_rng(4)
    keep = rng.random(len(rec["skx"])) < 0.7
    rec = {k: np.ascontiguousarray(v[keep]) for k, v in rec.items()}
    n = len(rec["skx"])
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    _, ngw, whole = space.group_best(pc, G.Records.from_numpy(rec))
    want = [(g.first, g.count, g.best_index, g.h2d_bytes, g.d2h_bytes) for g in whole]
    P = oracle_problem(O, c["skeletons"])
    f, cnt, bi, bt = P.group_best(rec)
    assert want == [(int(f[g]), int(cnt[g]), int(bi[g]), want[g][3], want[g][4])
                    for g in range(len(f))]
    for world in (2, 3, 8, 64):
        bounds = [D.shard_range(n, r, world) for r in range(world)]
        infos, locals_ = [], []
        for lo, hi in bounds:
            part = {k: np.ascontiguousarray(v[lo:hi]) for k, v in rec.items()}
            _, ng, gs = space.group_best(pc, G.Records.from_numpy(part), index_base=lo)
            keys = [D.record_key(*[part[k][i] for k in ("skx", "nx", "ny", "iters")])
                    for i in (0, hi - lo - 1)]
            infos.append((hi - lo, keys[0], keys[1], gs[0], gs[-1], len(gs)))
            locals_.append(gs)
        fix = D.shard_group_fixups(infos)
        got = []
        for r in range(world):
            got += [(g.first, g.count, g.best_index, g.h2d_bytes, g.d2h_bytes)
                    for g in D.apply_group_fixup(locals_[r], fix[r])]
        assert got == want, world
