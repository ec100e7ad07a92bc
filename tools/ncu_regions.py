"""Aggregate ncu source-view stall samples (cuda,sass view) by file/line region.

usage: python tools/ncu_regions.py <src_cs.csv>   (from: ncu -i rep --page source --csv --print-source cuda,sass)
Regions for kb1_v4: point physics (pointwise.cuh), PW stage C (kb1_v4.cuh pw_point), KW (the rest)."""
import csv
import sys
from collections import defaultdict


def region(path, line):
    f = path.rsplit('/', 1)[-1]
    if f == 'pointwise.cuh':
        return 'PW point_eval'
    if f == 'kb1_v4.cuh':
        if 414 <= line <= 513 or 540 <= line <= 569:
            return 'PW stageC/io'
        return 'KW'
    return 'KW(helpers:' + f + ')'


def main(fn):
    rows = list(csv.reader(open(fn)))
    path, hdr = None, None
    agg = defaultdict(lambda: defaultdict(float))
    for r in rows:
        if not r:
            continue
        if r[0] == 'File Path':
            path = r[1]
            continue
        if r[0] == 'Function Name':
            continue
        if r[0] == 'Line No':
            hdr = {h: i for i, h in enumerate(r) if h != 'Source'}
            hdr['Address'] = r.index('Address')
            continue
        if hdr is None or len(r) < 5:
            continue
        try:
            line = int(r[0])
        except ValueError:
            continue
        g = region(path, line)
        for k, i in hdr.items():
            if (k.startswith('stall_') and '(Not Issued)' not in k) or k in ('Warp Stall Sampling (All Samples)', 'Instructions Executed'):
                try:
                    agg[g][k] += float(r[i] or 0)
                except ValueError:
                    pass
    tot = sum(a['Warp Stall Sampling (All Samples)'] for a in agg.values())
    for g, a in sorted(agg.items(), key=lambda x: -x[1]['Warp Stall Sampling (All Samples)']):
        s = a['Warp Stall Sampling (All Samples)']
        top = sorted(((k, v) for k, v in a.items() if k.startswith('stall_')), key=lambda x: -x[1])[:8]
        print(f"{g:32s} samples {100*s/tot:5.1f}%  inst {a['Instructions Executed']:.3e}  " +
              ' '.join(f"{k[6:]}={100*v/max(s,1):.0f}%" for k, v in top))


if __name__ == '__main__':
    main(sys.argv[1])
