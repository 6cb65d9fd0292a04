"""Debug aid: time eval/best of a C3s prefix on the GPU (canonical tiles)."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
from paper_conf_ipps_boyermk13_b200 import build as B
B.build()
from paper_conf_ipps_boyermk13_b200 import grophecy as G
from synth import records as R, skeletons as S
name = sys.argv[1] if len(sys.argv) > 1 else "c3s"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
c = R.config(name)
import numpy as np
if len(sys.argv) > 3 and sys.argv[3] == "slice":
    idx = np.concatenate([np.arange(k * c["n"] // 64, k * c["n"] // 64 + n, dtype=np.uint64)
                          for k in range(64)])
    rec = R.gen_records_at(c, idx)
else:
    rec = R.gen_records(c, 0, n)
pc = G.pcie(G.fit_pcie(S.PAPER_TS, S.PAPER_TL, S.PAPER_SL))
sp = G.Space(c["skeletons"], S.FX5600)
t0 = time.time()
h, d, t = sp.eval(pc, G.Records.from_numpy(rec))
torch.cuda.synchronize()
print("eval", n, time.time() - t0, flush=True)
t0 = time.time()
rc, b = sp.best(pc, G.Records.from_numpy(rec))
print("best", n, time.time() - t0, b.index, flush=True)
