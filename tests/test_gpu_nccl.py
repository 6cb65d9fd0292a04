"""The C-ABI cross-GPU min-loc (grophecy_best_allreduce) with a
single-rank NCCL communicator on the one GPU this environment has: the
all-gather + combine path must return exactly grophecy_best's result (the
multi-rank combine itself is covered by the host and gloo tests)."""
import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import oracle_problem, paper_pcie

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


def test_single_rank_allreduce_equals_best(G, O):
    c = R.config("c3")
    pc = paper_pcie(G)
    space = G.Space(c["skeletons"], S.FX5600)
    comm = G.NcclComm(1, 0, G.nccl_unique_id(), 0)
    try:
        for lo, n in ((0, 100_000), (1_000_003, 65_537)):
            rec = R.gen_records(c, lo, lo + n)
            dev = G.Records.from_numpy(rec)
            rc1, b1 = space.best(pc, dev, index_base=lo)
            rc2, b2 = space.best_allreduce(pc, dev, comm, index_base=lo)
            assert rc1 == rc2 and b1.as_tuple() == b2.as_tuple()
            orc, ob = oracle_problem(O, c["skeletons"]).best(rec, index_base=lo)
            assert (b2.index, b2.t_total_s) == (ob.index, ob.t_total_s)
    finally:
        comm.close()
        space.close()
