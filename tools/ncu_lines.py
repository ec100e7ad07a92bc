"""Per-CUDA-source-line stall samples and executed instructions from an ncu report (needs -lineinfo)."""
import csv
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
fname = None
agg = defaultdict(lambda: [0.0, 0.0, ''])
tot = 0.0
hdr = None
for r in rows:
    if r and r[0] == 'File Path':
        fname = r[1].split('/')[-1]
        continue
    if r and r[0] == 'Line No':
        hdr = r
        continue
    if not hdr or len(r) != len(hdr) or r[0] == '':
        continue
    key = (fname, int(r[0]))
    f = lambda x: float(x) if x not in ("", "-") else 0.0
    s = f(r[4])
    agg[key][0] += s
    agg[key][1] += f(r[7])
    agg[key][2] = r[1][:90]
    tot += s
print('total stall samples', tot)
for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{k[0]:22s}:{k[1]:<4d} {100*v[0]/tot:5.1f}%  inst {v[1]:.2e}  {v[2]}")
