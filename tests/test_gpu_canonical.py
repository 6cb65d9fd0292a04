"""GPU parity on canonical tiles (512 records = 32 design points x 16
transformations, one skeleton): the fast pass-1 kernel for
every output — eval, eval_parts (t_iter, t_once, t_h2d, t_d2h) and best —
including run-once kernels, infeasible (kernel, transformation) pairs in the
per-iteration and in the run-once sum, and a ragged tail left to pass 2."""
import copy
import math

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import assert_same, oracle_problem, paper_pcie, records_slice

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


def _segment(c, s, n):
    """n consecutive records of skeleton s's C4 segment, from a group boundary."""
    G_ = c["n"] // 16
    lo = -(-s * G_ // 16) * 16
    return records_slice(c, np.arange(lo, lo + n, dtype=np.uint64))


def _parts_parity(G, O, skels, rec):
    space = G.Space(skels, S.FX5600)
    pc = paper_pcie(G)
    out = space.eval_parts(pc, G.Records.from_numpy(rec))
    torch.cuda.synchronize()
    h, d, t, ti, to, th, td = [o.cpu().numpy() for o in out]
    P = oracle_problem(O, skels)
    for k in range(len(rec["skx"])):
        a = [int(rec[f][k]) for f in ("skx", "nx", "ny", "iters")]
        ok, parts = P.eval_parts_one(*a)
        assert ok
        assert _bits([ti[k], to[k], th[k], td[k]]).tolist() == _bits(parts).tolist(), (k, a)
    o = P.eval(rec)
    assert_same((h.view(np.uint64), d.view(np.uint64), t), o)
    rc, b = space.best(pc, G.Records.from_numpy(rec))
    orc, ob = P.best(rec)
    assert (b.index, b.n_valid) == (ob.index, ob.n_valid)
    if ob.index != G.UINT64_MAX:
        assert _bits([b.t_total_s]) == _bits([ob.t_total_s])
        assert (b.h2d_bytes, b.d2h_bytes) == (ob.h2d_bytes, ob.d2h_bytes)
    space.close()
    return t


@pytest.mark.parametrize("s", range(16))
def test_eval_parts_canonical_every_c4_skeleton(G, O, s):
    c = R.config("c4")
    rec = _segment(c, s, 2 * 512 + 37)      # two canonical tiles + a ragged tail
    _parts_parity(G, O, c["skeletons"], rec)


def test_infeasible_pairs_in_both_sums(G, O):
    """CFD (one run-once kernel) and a variant with two run-once kernels;
    transformation 3: run-once kernel infeasible; 5: a per-iteration kernel
    infeasible; 7: both (occupancy 0: tpb above max_threads_per_block)."""
    c = R.config("c4")
    cfd = copy.deepcopy(c["skeletons"][4])
    assert cfd["name"] == "cfd" and not cfd["kernels"][0]["per_iter"]
    for x, ks in ((3, (0,)), (5, (2,)), (7, (0, 3))):
        for k in ks:
            cfd["kx"][x][k]["tpb"] = 2 * S.FX5600["max_threads_per_block"]
    cfd2 = copy.deepcopy(cfd)
    cfd2["name"] = "cfd_two_once"
    cfd2["kernels"][2]["per_iter"] = False
    rec = _segment(c, 4, 4 * 512 + 5)
    skel = np.zeros(len(rec["skx"]), np.uint32)
    skel[1024:] = 1                          # tiles 0-1: cfd, tiles 2-3 (+ tail): cfd2
    rec["skx"] = (skel << 16) | (rec["skx"] & 0xffff)
    t = _parts_parity(G, O, [cfd, cfd2], rec)
    x = rec["skx"] & 0xffff
    assert np.all(np.isinf(t[np.isin(x, (3, 5, 7))]))
    assert np.isfinite(t).sum() >= len(t) // 2   # the others stay mostly feasible


def test_canonical_tiles_with_invalid_record(G, O):
    """One invalid record spoils its tile (general path); its neighbours stay
    canonical; outputs and best are unchanged elsewhere."""
    c = R.config("c4")
    rec = _segment(c, 9, 3 * 512)
    rec["iters"][512 + 100] = 0
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    P = oracle_problem(O, c["skeletons"])
    h, d, t = space.eval(pc, G.Records.from_numpy(rec))
    torch.cuda.synchronize()
    o = P.eval(rec)
    assert_same((h.cpu().numpy().view(np.uint64), d.cpu().numpy().view(np.uint64),
                 t.cpu().numpy()), o)
    assert math.isnan(t[612].item())
    rc, b = space.best(pc, G.Records.from_numpy(rec))
    orc, ob = P.best(rec)
    assert rc == G.EBADCAND and (b.index, b.n_invalid) == (ob.index, ob.n_invalid) == (ob.index, 1)
    space.close()


@pytest.mark.parametrize("start", [333_333_333, 125_000_003])
def test_shard_starting_inside_a_group(G, O, start):
    """A shard boundary inside a design point (P = 3 shards of 10^9): the
    head up to the next multiple of 16 is projected on its own, the rest in
    canonical tiles; eval and best (global indices) match the oracle."""
    c = R.config("c4")
    rec = records_slice(c, np.arange(start, start + 3 * 512 + 40, dtype=np.uint64))
    space = G.Space(c["skeletons"], S.FX5600)
    pc = paper_pcie(G)
    P = oracle_problem(O, c["skeletons"])
    h, d, t = space.eval(pc, G.Records.from_numpy(rec), index_base=start)
    torch.cuda.synchronize()
    assert_same((h.cpu().numpy().view(np.uint64), d.cpu().numpy().view(np.uint64),
                 t.cpu().numpy()), P.eval(rec))
    rc, b = space.best(pc, G.Records.from_numpy(rec), index_base=start)
    orc, ob = P.best(rec, index_base=start)
    assert (b.index, b.n_valid) == (ob.index, ob.n_valid)
    assert _bits([b.t_total_s]) == _bits([ob.t_total_s])
    space.close()


@pytest.mark.parametrize("n", [16, 160, 512 + 48, 3 * 512 + 496])
def test_partial_canonical_tail(G, O, n):
    """A batch ending in whole design points short of a full tile: the last
    tile is canonical with fewer than 32 design points (lanes past them stand
    in for the first and output nothing)."""
    c = R.config("c4")
    for s in (1, 4, 9):
        _parts_parity(G, O, c["skeletons"], _segment(c, s, n))
