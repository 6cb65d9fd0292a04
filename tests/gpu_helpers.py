"""Helpers for the GPU parity tests: run the CUDA path through the C ABI and
the oracle on the same seeded records, compare element by element."""
import numpy as np

from synth import records as R
from synth import skeletons as S


def paper_pcie(G):
    return G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))


def oracle_problem(O, skels, gpu=S.FX5600):
    rc, link = O.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL)
    return O.Problem(skels, gpu, link)


def gpu_eval(G, space, pc, rec_np, index_base=0):
    rec = G.Records.from_numpy(rec_np)
    h, d, t = space.eval(pc, rec, index_base=index_base)
    import torch
    torch.cuda.synchronize()
    return (h.cpu().numpy().view(np.uint64), d.cpu().numpy().view(np.uint64),
            t.cpu().numpy())


def assert_same(gpu, ora, idx=None):
    """Bit-exact bytes; bitwise-equal times (NaN positions equal)."""
    gh, gd, gt = gpu
    oh, od, ot = ora
    if idx is not None:
        gh, gd, gt = gh[idx], gd[idx], gt[idx]
    bad = np.nonzero(gh != oh)[0]
    assert bad.size == 0, f"h2d mismatch at {bad[:10]}: {gh[bad[:5]]} vs {oh[bad[:5]]}"
    bad = np.nonzero(gd != od)[0]
    assert bad.size == 0, f"d2h mismatch at {bad[:10]}: {gd[bad[:5]]} vs {od[bad[:5]]}"
    gb = gt.view(np.uint64)
    ob = ot.view(np.uint64)
    nan = np.isnan(gt) & np.isnan(ot)
    bad = np.nonzero((gb != ob) & ~nan)[0]
    if bad.size:
        rel = np.abs(gt[bad] - ot[bad]) / np.abs(ot[bad])
        raise AssertionError(f"time mismatch at {bad.size} records, first {bad[:5]}: "
                             f"{gt[bad[:5]]} vs {ot[bad[:5]]}, max rel {np.nanmax(rel)}")


def records_slice(cfg, idx):
    """Oracle-side records for arbitrary global indices."""
    return R.gen_records_at(cfg, np.asarray(idx, dtype=np.uint64))
