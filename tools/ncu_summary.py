"""Summarize an ncu --set full report: key metrics + SASS opcode mix / stall samples."""
import csv
import json
import subprocess
import sys
from collections import defaultdict

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'launch__occupancy_limit_registers', 'launch__occupancy_limit_shared_mem',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum', 'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum',
        'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'smsp__sass_thread_inst_executed_op_dfma_pred_on.sum', 'smsp__sass_thread_inst_executed_op_dadd_pred_on.sum',
        'smsp__sass_thread_inst_executed_op_dmul_pred_on.sum', 'sass__inst_executed_local_loads',
        'sm__cycles_elapsed.avg', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed',
        'smsp__warps_issue_stalled_barrier_per_warp_active.pct', 'smsp__warps_issue_stalled_short_scoreboard_per_warp_active.pct',
        'smsp__warps_issue_stalled_wait_per_warp_active.pct', 'smsp__warps_issue_stalled_math_pipe_throttle_per_warp_active.pct',
        'smsp__warps_issue_stalled_mio_throttle_per_warp_active.pct', 'smsp__warps_issue_stalled_long_scoreboard_per_warp_active.pct',
        'smsp__warps_issue_stalled_not_selected_per_warp_active.pct', 'smsp__warps_issue_stalled_selected_per_warp_active.pct',
        'smsp__warps_issue_stalled_dispatch_stall_per_warp_active.pct', 'smsp__warps_issue_stalled_lg_throttle_per_warp_active.pct']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for i, h in enumerate(hdr):
            if h in KEYS or h in ('Kernel Name',):
                d[h] = (vals[i], units[i])
        res.append(d)
    return res


def sass_mix(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr = rows[1]
    idx = {h: j for j, h in enumerate(hdr)}
    S = 'Warp Stall Sampling (All Samples)'
    agg = defaultdict(lambda: [0.0, 0.0])
    tot = 0.0
    for r in rows[2:]:
        if len(r) != len(hdr):
            continue
        toks = r[1].split()
        if not toks:
            continue
        op = toks[1] if toks[0].startswith('@') and len(toks) > 1 else toks[0]
        op = op.split('.')[0]
        agg[op][0] += float(r[idx['Instructions Executed']] or 0)
        agg[op][1] += float(r[idx[S]] or 0)
        tot += float(r[idx[S]] or 0)
    return {k: {'warp_inst': v[0], 'stall_pct': round(100 * v[1] / max(tot, 1), 2)}
            for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[:20]}


if __name__ == '__main__':
    rep = sys.argv[1]
    r = raw(rep)
    for d in r:
        for k in KEYS:
            if k in d:
                print(f"{k:80s} {d[k][0]:>20s} {d[k][1]}")
    mix = sass_mix(rep)
    for k, v in mix.items():
        print(f"{k:10s} {v['warp_inst']:.3e} {v['stall_pct']}%")
    if len(sys.argv) > 2:
        json.dump({'metrics': r, 'sass_mix': mix}, open(sys.argv[2], 'w'), indent=1)
