"""Top source lines of an ncu report by executed instructions and stall samples."""
import csv
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
hdr = None
lines = []
for r in rows:
    if r and r[0] == 'Line No':
        hdr = r
        continue
    if hdr and r and r[0] not in ('',) and r[0].isdigit():
        d = dict(zip(hdr, r))
        try:
            ins = int(d['Instructions Executed'])
            st = int(d['Warp Stall Sampling (All Samples)'])
        except (ValueError, KeyError):
            continue
        lines.append((int(r[0]), r[1][:90], ins, st))
tot_i = sum(l[2] for l in lines) or 1
tot_s = sum(l[3] for l in lines) or 1
print(f'total instr {tot_i}, samples {tot_s}')
print('-- by instructions')
for l in sorted(lines, key=lambda x: -x[2])[:n]:
    print(f'{l[0]:5d} {100*l[2]/tot_i:5.1f}% {100*l[3]/tot_s:5.1f}%  {l[1]}')
print('-- by stall samples')
for l in sorted(lines, key=lambda x: -x[3])[:n]:
    print(f'{l[0]:5d} {100*l[2]/tot_i:5.1f}% {100*l[3]/tot_s:5.1f}%  {l[1]}')
