"""Print the warp-stall breakdown (per issued instruction) of an ncu --set full report."""
import csv
import subprocess
import sys

out = subprocess.run(['ncu', '-i', sys.argv[1], '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[0]
for v in rows[2:]:
    print(v[h.index('Kernel Name')][:60])
    items = []
    for i, k in enumerate(h):
        if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('_per_issue_active.ratio'):
            try:
                items.append((float(v[i]), k[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]))
            except ValueError:
                pass
    for val, name in sorted(items, reverse=True):
        if val > 0.05:
            print(f"  {name:24s} {val:.2f}")
