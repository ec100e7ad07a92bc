"""Stall samples and executed instructions of an ncu report grouped by source-line ranges of one file.

usage: python tools/ncu_stage_split.py <report.ncu-rep> <file.cuh> name:lo-hi [name:lo-hi ...]
Lines of other files (pointwise.cuh, table accessors) are reported per file."""
import csv
import subprocess
import sys
from collections import defaultdict

rep, target = sys.argv[1], sys.argv[2]
ranges = []
for spec in sys.argv[3:]:
    name, lh = spec.split(':')
    lo, hi = lh.split('-')
    ranges.append((name, int(lo), int(hi)))
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
agg = defaultdict(lambda: [0.0, 0.0])
fname, hdr, tot = None, None, 0.0
for r in rows:
    if r and r[0] == 'File Path':
        fname = r[1].split('/')[-1]
        continue
    if r and r[0] == 'Line No':
        hdr = r
        continue
    if not hdr or len(r) != len(hdr) or r[0] == '':
        continue
    f = lambda x: float(x) if x not in ("", "-") else 0.0
    line = int(r[0])
    key = fname
    if fname == target:
        key = f'{target}:other'
        for name, lo, hi in ranges:
            if lo <= line <= hi:
                key = name
                break
    agg[key][0] += f(r[4])
    agg[key][1] += f(r[7])
    tot += f(r[4])
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{k:28s} {100 * v[0] / tot:5.1f}%  inst {v[1]:.3e}")
