"""Striped batches and the multi-GPU partition on one device.

* The stripe map of grophecy_batch (include/grophecy.h): a rank's stripes
  stored back to back and projected by one launch report the same global
  best as the contiguous records (ties resolve to the lowest global index:
  the map is increasing).
* The bench's N > 1 partition (dist.stripe_layout, every rank = one striped
  batch + a contiguous tail): for P = 2, 3, 8 ranks simulated on one GPU, the
  min-loc of the ranks' results equals the oracle's full-size golden best
  (tests/golden/c4_full.json, c3_full.json: scripts/oracle_golden.py).
* A real two-process run (torch.distributed gloo, both ranks on cuda:0)
  drives the GPU path end to end and returns the golden best.
* grophecy_best_host with the stripe map (the e2e path) agrees.
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import oracle_problem, paper_pcie

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)


@pytest.fixture(scope="module")
def G():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy
    torch.cuda.set_device(0)
    return grophecy


def golden_best(name):
    return json.load(open(os.path.join(HERE, "golden", f"{name}_full.json")))["total"]


def rank_share(G, D, cfg, rank, world, stripes):
    """The records and batches of rank `rank` in the bench's N > 1 layout."""
    N = cfg["n"]
    L, n_main, (t_lo, t_hi) = D.stripe_layout(N, rank, world, stripes)
    n_local = n_main + t_hi - t_lo
    rec = G.Records.empty(n_local)
    for k in range(n_main // L if L else 0):
        part = G.Records(*[t[k * L:(k + 1) * L] for t in (rec.skx, rec.nx, rec.ny, rec.iters)])
        G.synth_records(cfg, rank * L + k * world * L, L, out=part)
    if t_hi > t_lo:
        part = G.Records(*[t[n_main:] for t in (rec.skx, rec.nx, rec.ny, rec.iters)])
        G.synth_records(cfg, t_lo, t_hi - t_lo, out=part)
    batches = []
    if n_main:
        batches.append(rec.batch(index_base=rank * L, start=0, stop=n_main, stripe_len=L,
                                 stripe_stride=world * L))
    if t_hi > t_lo or not batches:
        batches.append(rec.batch(index_base=t_lo, start=n_main, stop=n_local))
    return rec, batches


@pytest.mark.parametrize("name,world,stripes", [("c3", 2, 4), ("c3", 3, 5), ("c4", 8, 16),
                                                ("c4", 2, 16)])
def test_partition_matches_golden(G, name, world, stripes):
    from paper_conf_ipps_boyermk13_b200 import dist as D
    cfg = R.config(name)
    gold = golden_best(name)
    pc = paper_pcie(G)
    space = G.Space(cfg["skeletons"], S.FX5600)
    res = G.best_result_tensor(world)
    covered = 0
    for r in range(world):
        rec, batches = rank_share(G, D, cfg, r, world, stripes)
        covered += rec.n
        for k, b in enumerate(batches):
            space.best_async(pc, b, res[6 * r:6 * r + 6], accumulate=k > 0)
        del rec
        torch.cuda.synchronize()
    assert covered == cfg["n"]
    out = G.best_result_tensor(1)
    G.best_combine(res, world, out)
    b = G.result_from_tensor(out)
    assert b.index == gold["best_index"]
    assert int(np.array([b.t_total_s]).view(np.uint64)[0]) == gold["best_t_bits"]
    assert (b.n_valid, b.n_invalid) == (gold["n_valid"], gold["n_invalid"])
    space.close()


def test_stripe_map_ties_and_oracle(G, O):
    """Tiny striped batch with exact ties (App. B.2 HotSpot: xforms 0/8/12
    tie): stripes of 16 records (one design point each) at stride 48 — the
    lowest global index among the tied candidates wins, as the oracle says
    for the same global records."""
    sk = [S.s1_hotspot()]
    pc = paper_pcie(G)
    space = G.Space(sk, S.FX5600)
    # global workload: 3 * 4 stripes of 16 records, each record = (x, 1024^2, 10)
    n_glob = 16 * 12
    gx = np.arange(n_glob) % 16
    glob = {"skx": gx.astype(np.uint32), "nx": np.full(n_glob, 1024, np.uint32),
            "ny": np.full(n_glob, 1024, np.uint32), "iters": np.full(n_glob, 10, np.uint32)}
    # rank 1 of 3: stripes j = 1 + 3 k -> global [16 j, 16 j + 16)
    idx = np.concatenate([np.arange(16 * j, 16 * j + 16) for j in (1, 4, 7, 10)])
    local = {k: v[idx] for k, v in glob.items()}
    rec = G.Records.from_numpy(local)
    rc, b = space.best(pc, rec, batch=rec.batch(index_base=16, stripe_len=16, stripe_stride=48))
    P = oracle_problem(O, sk)
    orc, ob = P.best(local)          # local order: same argmin position
    assert b.index == 16 + (ob.index // 16) * 48 + ob.index % 16
    assert b.t_total_s == ob.t_total_s
    # the e2e host path with the same stripe map
    host = {k: torch.from_numpy(v.view(np.int32)).pin_memory() for k, v in local.items()}
    rc2, b2 = space.best_host(pc, host, index_base=16, stripe_len=16, stripe_stride=48)
    assert b2.as_tuple() == b.as_tuple()
    # invalid stripe map
    from paper_conf_ipps_boyermk13_b200.grophecy import GrophecyError
    with pytest.raises(GrophecyError):
        space.best(pc, rec, batch=rec.batch(index_base=0, stripe_len=32, stripe_stride=16))
    space.close()


def test_two_process_gloo_run(G):
    """bench.py's N = 2 path with two real processes on one GPU (gloo
    collectives: NCCL needs one GPU per rank) returns the golden C4 best."""
    env = dict(os.environ, GROPHECY_DIST_BACKEND="gloo", MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29533", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "2", "--warmup", "1", "--no-cpu-baseline", "--no-e2e"]
    out = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    line = json.loads([ln for ln in out.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2
    assert line["best"]["index"] == golden_best("c4")["best_index"]
