"""Full-size parity: the CUDA path at BASELINE.json's full sizes against the
oracle's goldens (``tests/golden/<cfg>_full.json``, written by
``scripts/oracle_golden.py``, which imports only ``oracle/`` and ``synth/``).

For C2 (10^6), C3 (10^7) and C4 (10^9 records), in the launch configuration
bench.py times (device-generated records, one fused best launch over the whole
batch):

* the fused argmin (index, t bits, bytes, n_valid / n_invalid) equals the
  oracle's global best ("best achievable performance";
  N7 ties -> lowest global index);
* per shard (16 for C4): the best over the shard's record range equals the
  oracle's shard best (the multi-GPU partition);
* order-independent checksums over EVERY record's eval outputs equal the
  oracle's: sum of H2D / D2H bytes (mod 2^64), XOR and sum (mod 2^64) of the
  binary64 bit patterns of t over the valid records, counts of valid,
  invalid and infeasible (+inf) records.
"""
import json
import os

import numpy as np
import pytest

from synth import records as R
from synth import skeletons as S
from tests.gpu_helpers import paper_pcie

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

HERE = os.path.dirname(os.path.abspath(__file__))
M64 = (1 << 64) - 1


@pytest.fixture(scope="module")
def G():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_boyermk13_b200 import build
    build.build()
    from paper_conf_ipps_boyermk13_b200 import grophecy
    torch.cuda.set_device(0)
    return grophecy


def golden(name):
    p = os.path.join(HERE, "golden", f"{name}_full.json")
    if not os.path.exists(p):
        pytest.fail(f"missing golden {p} (run scripts/oracle_golden.py {name})")
    doc = json.load(open(p))
    assert doc["total"] is not None, "golden incomplete"
    return doc


def _sum64(x):
    """sum mod 2^64 of an int64 tensor's two's-complement values (exact:
    32-bit halves summed separately in int64)."""
    lo = (x & 0xFFFFFFFF).sum().item()
    hi = ((x >> 32) & 0xFFFFFFFF).sum().item()
    return (lo + (hi << 32)) & M64


def _xor64(x):
    """XOR-reduce an int64 tensor by pairwise folding."""
    while x.numel() > 1:
        if x.numel() & 1:
            x = torch.cat([x, torch.zeros(1, dtype=x.dtype, device=x.device)])
        x = x[0::2] ^ x[1::2]
    return int(x.item()) & M64 if x.numel() else 0


def _u64(v):
    return int(v) & M64


def check_full(G, name, chunk=1 << 24):
    doc = golden(name)
    c = R.config(name)
    N = c["n"]
    assert doc["n"] == N
    pc = paper_pcie(G)
    space = G.Space(c["skeletons"], S.FX5600)
    dev = G.synth_records(c)
    # ---- global fused argmin (bench launch configuration) ----
    rc, b = space.best(pc, dev)
    tot = doc["total"]
    assert b.index == tot["best_index"]
    assert _u64(np.array([b.t_total_s]).view(np.uint64)[0]) == tot["best_t_bits"]
    assert (b.h2d_bytes, b.d2h_bytes) == (tot["best_h2d"], tot["best_d2h"])
    assert (b.n_valid, b.n_invalid) == (tot["n_valid"], tot["n_invalid"])
    # ---- per shard ----
    for sh in doc["shards"]:
        lo, hi = sh["lo"], sh["hi"]
        rc, bs = space.best(pc, dev, batch=dev.batch(index_base=lo, start=lo, stop=hi))
        assert bs.index == sh["best_index"], (lo, hi)
        assert _u64(np.array([bs.t_total_s]).view(np.uint64)[0]) == sh["best_t_bits"]
    # ---- checksums over every record's eval outputs ----
    eh = torch.empty(chunk, dtype=torch.int64, device="cuda")
    ed = torch.empty(chunk, dtype=torch.int64, device="cuda")
    et = torch.empty(chunk, dtype=torch.float64, device="cuda")
    acc = {"sum_h2d": 0, "sum_d2h": 0, "sum_t_bits": 0, "xor_t_bits": 0,
           "n_valid": 0, "n_invalid": 0, "n_inf": 0}
    for s in range(0, N, chunk):
        e = min(N, s + chunk)
        sub = G.Records(dev.skx[s:e], dev.nx[s:e], dev.ny[s:e], dev.iters[s:e])
        h, d, t = eh[:e - s], ed[:e - s], et[:e - s]
        space.eval(pc, sub, index_base=s, out=(h, d, t))
        valid = ~torch.isnan(t)
        bits = t.view(torch.int64)[valid]
        acc["sum_h2d"] = (acc["sum_h2d"] + _sum64(h)) & M64
        acc["sum_d2h"] = (acc["sum_d2h"] + _sum64(d)) & M64
        acc["sum_t_bits"] = (acc["sum_t_bits"] + _sum64(bits)) & M64
        acc["xor_t_bits"] ^= _xor64(bits)
        nv = int(valid.sum().item())
        acc["n_valid"] += nv
        acc["n_invalid"] += (e - s) - nv
        acc["n_inf"] += int(torch.isinf(t).sum().item())
    space.invalid_count()   # reset the device flag counter
    for k, v in acc.items():
        assert v == tot[k], (k, v, tot[k])
    space.close()


def test_c2_full_golden(G):
    check_full(G, "c2")


def test_c3_full_golden(G):
    check_full(G, "c3")


def test_c4_full_golden(G):
    check_full(G, "c4")
