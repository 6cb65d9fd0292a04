"""Instructions / stall samples of an ncu capture grouped by source ranges of
project.cu (phases of the sweep kernel).  usage: ncu_groups.py REP"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
REASONS = ['stall_wait', 'stall_barrier', 'stall_long_sb', 'stall_short_sb', 'stall_math',
           'stall_dispatch', 'stall_branch_resolving', 'stall_selected', 'stall_not_selected']
hdr, L = None, []
for r in rows:
    if r and r[0] == 'Line No':
        hdr = r
        continue
    if hdr and r and r[0].isdigit():
        d = dict(zip(hdr, r))
        try:
            L.append((int(r[0]), int(d['Instructions Executed']), int(d['Warp Stall Sampling (All Samples)']),
                      {k: int(d[k]) for k in REASONS}))
        except (ValueError, KeyError):
            pass
src = open('paper_conf_ipps_boyermk13_b200/csrc/project.cu').read().splitlines()


def find(pat, after=0):
    for i, l in enumerate(src):
        if i >= after and pat in l:
            return i + 1
    return 10 ** 9


# regions of project.cu in file order (each runs to the next mark)
MARKS = [('helpers', '__device__ __forceinline__ long long aff8n'),
         ('usage_fn', '__device__ __forceinline__ void group_usage('),
         ('other', '// ---- 1-D bulk copies'),
         ('usage_fn', 'template <bool U32>   // every partial sum below 2^32'),
         ('other', '// CTA tile copy (thread 0)'),
         ('phaseA', 'template <int CXT, unsigned long long ROW>'),
         ('cls_times', '// Saturated kernel times of NCH'),
         ('other', '// Transfer bytes of a design point'),
         ('prologue', 'sweep_kernel(const Params P)'),
         ('phaseC', '// ---- C: tile r, CTA-wide'),
         ('totals', '// totals (P:L77, L147, L167)'),
         ('phaseA_task', '// ---- A/B tasks of tile r + 1'),
         ('phaseB', '// ---- B: work counts and usage of design point g'),
         ('round_end', 'PT_MARK(3);   // phase B'),
         ('pass2', '// ---- pass 2 in the same (cooperative) launch'),
         ('other', '// Pass 2: the listed tiles as general')]
marks, pos = [], 0
for n, p in MARKS:
    pos = find(p, pos)
    marks.append((pos, n))
ti = sum(x[1] for x in L) or 1
ts = sum(x[2] for x in L) or 1
acc = {}
for ln, i, s, rs in L:
    name = 'other'
    for lo, n in marks:
        if ln >= lo:
            name = n
    a = acc.setdefault(name, [0, 0, {k: 0 for k in REASONS}])
    a[0] += i
    a[1] += s
    for k in REASONS:
        a[2][k] += rs[k]
n_cand = float(sys.argv[2]) if len(sys.argv) > 2 else 1e9
for k, (i, s, rs) in sorted(acc.items(), key=lambda x: -x[1][0]):
    print(f"{k:10s} instr {100 * i / ti:5.1f}%  {32 * i / n_cand:6.1f} thread-instr/cand  stalls {100 * s / ts:5.1f}%  " +
          " ".join(f"{r[6:]}={100 * v / ts:.1f}" for r, v in rs.items() if v > 0.004 * ts))
