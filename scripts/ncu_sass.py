"""Hot SASS instructions of an ncu report (source page, sass view):
executed-instruction share, stall-sample share and the top stall reasons.

    python scripts/ncu_sass.py report.ncu-rep [min_frac_of_max]
"""
import csv
import subprocess
import sys

rep = sys.argv[1]
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.3
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
hdr = rows[1]
L = []
for r in rows[2:]:
    d = dict(zip(hdr, r))
    try:
        L.append((d['Address'][-5:], d['Source'].strip(), int(d['Instructions Executed'] or 0),
                  int(d['Warp Stall Sampling (All Samples)'] or 0), d))
    except (ValueError, KeyError):
        pass
tot_i = sum(x[2] for x in L) or 1
tot_s = sum(x[3] for x in L) or 1
mx = max(x[2] for x in L)
stall_cols = [c for c in hdr if c.startswith('stall_') or 'Stall' in c and c not in (
    'Warp Stall Sampling (All Samples)', 'Warp Stall Sampling (Not-issued Samples)')]
print(f'total instr {tot_i}, samples {tot_s}')
for a, s, i, st, d in L:
    if i >= frac * mx:
        top = sorted(((int(d[c] or 0) if d[c].isdigit() else 0, c) for c in stall_cols), reverse=True)[:2]
        tops = ' '.join(f'{c[:18]}={v}' for v, c in top if v)
        print(f'{a} {100*i/tot_i:5.2f}% {100*st/tot_s:5.2f}%  {s[:60]:60s} {tops}')
