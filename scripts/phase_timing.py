"""Per-phase time of the sweep kernel on C4 (diagnostic build with
GROPHECY_PHASE_TIMING=1): warp-cycles per phase, summed over warps, as
fractions.  usage: GROPHECY_PHASE_TIMING=1 python -m ...build --force;
python scripts/phase_timing.py"""
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ipps_boyermk13_b200 import grophecy as G  # noqa: E402
from synth import records as R  # noqa: E402
from synth import skeletons as S  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c4"
cfg = R.config(name)
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
space = G.Space(cfg["skeletons"], S.FX5600)
seg = os.environ.get("SEG_ONLY")   # one skeleton's segment (as scripts/segbench.py)
if seg is not None:
    ns, Gn = len(cfg["skeletons"]), (cfg["n"] + 15) // 16
    s = int(seg)
    lo = -(-s * Gn // ns) * 16
    hi = min(cfg["n"], -(-(s + 1) * Gn // ns) * 16)
    rec = G.synth_records(cfg, lo, min(hi - lo, 1 << 25))
    print("segment", s, cfg["skeletons"][s]["name"])
else:
    rec = G.synth_records(cfg)
space.best(pc, rec)
fn = G.lib().grophecy_debug_phase_cycles
fn.argtypes = [C.POINTER(C.c_uint64)]
out = (C.c_uint64 * 8)()
fn(out)
space.best(pc, rec)
torch.cuda.synchronize()
fn(out)
names = ["wait records (TMA)", "phase A", "table decision", "phase B", "wait A/B tasks (abar)", "phase C"]
tot = sum(out[i] for i in range(6))
for i, nm in enumerate(names):
    print(f"{nm:22s} {100 * out[i] / tot:6.2f} %")
