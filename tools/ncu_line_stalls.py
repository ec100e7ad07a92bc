#!/usr/bin/env python
"""Stall samples of one kernel per SOURCE LINE: ncu's SASS page (per-instruction stall reasons) matched to
the line table of the built library (nvdisasm -g), by instruction offset.  The report must come from the
same build as the library (checked: same instruction count and opcodes).

    python tools/ncu_line_stalls.py <report.ncu-rep> <mangled kernel name> [top]"""
import collections
import csv
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_dongdkrtd14_b200", "libblastcf.so")
COLS = ["Warp Stall Sampling (All Samples)", "stall_long_sb", "stall_barrier", "stall_wait", "stall_short_sb",
        "stall_math", "stall_mio", "stall_no_inst", "stall_branch_resolving"]


def line_table(kernel):
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "blast_cf.sm_100a.cubin", LIB], cwd=d, check=True, capture_output=True)
        sass = subprocess.run(["nvdisasm", "-c", "-g", os.path.join(d, "blast_cf.sm_100a.cubin")], capture_output=True,
                              text=True).stdout
    lines = sass.splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith(f".text.{kernel}:"))
    cur, tab = None, {}
    for l in lines[start + 1:]:
        if l.startswith(".text."):
            break
        m = re.search(r'//## File "([^"]+)", line (\d+)', l)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*)", l)
        if m:
            tab[int(m.group(1), 16)] = (cur, m.group(2).split(";")[0].strip())
    return tab


def main(rep, kernel, top=30):
    tab = line_table(kernel)
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, data = rows[1], rows[2:]
    ia, isrc = h.index("Address"), h.index("Source")
    base = int(data[0][ia], 16)
    if len(data) != len(tab):
        sys.exit(f"report has {len(data)} instructions, the library's {kernel} {len(tab)}: not the same build")
    idx = [h.index(c) for c in COLS]
    agg = collections.defaultdict(lambda: [0] * len(COLS))
    for r in data:
        li = tab[int(r[ia], 16) - base]
        if li[1].split()[0] != r[isrc].strip().split()[0]:
            sys.exit("opcode mismatch: not the same build")
        for j, i in enumerate(idx):
            agg[li[0]][j] += int(r[i] or 0)
    tot = [sum(v[j] for v in agg.values()) for j in range(len(COLS))]
    print("line".ljust(28), " ".join(c.replace("Warp Stall Sampling (All Samples)", "all").replace("stall_", "")[:9].rjust(9)
                                      for c in COLS))
    print("TOTAL".ljust(28), " ".join(str(t).rjust(9) for t in tot))
    for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print(f"{k[0]}:{k[1]}".ljust(28), " ".join(str(x).rjust(9) for x in v))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 30)
