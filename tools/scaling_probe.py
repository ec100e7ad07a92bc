#!/usr/bin/env python
"""Strong-scaling probe on ONE GPU (the NCCL path itself needs >= 2 GPUs).

For P = 1, 2, 4, 8 and the block partition bench.py uses (synth.partition), every rank's local mesh is
evaluated by itself on the whole GPU — a single-rank handle, no exchange — which is what one rank of a
P-GPU run computes (its KB1 over its zones, its KB2 over its nodes).  The compute-side strong-scaling
efficiency is E_c(P) = t(1) / (P * max_r t_r(P)); the exchange (shared-node rows + dt) comes on top,
hidden behind the interior zones by the overlap schedule (its message sizes are reported: the shared rows
per rank).  The loopback group (tests only) is not timed: it synchronizes the host once per rank for its
host-side min-dt, so its time says nothing about an NCCL run.

Every timed eval follows an L2 flush (a per-rank C4 working set at P = 8 is ~40 MB < L2): the worst case
for the small per-rank sizes.  Output: one JSON object on stdout.
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import argparse
    import torch
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--ranks", default="1,2,4,8")
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    stream = torch.cuda.Stream()
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    scratch = torch.empty(2 * l2 // 4, dtype=torch.float32, device=dev)
    m, s = synth.config(args.config, "S1")
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)

    def time_fn(fn, flush=True):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        tot = 0.0
        for _ in range(args.iters):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(stream):
                if flush:
                    scratch.fill_(1.0)
                a.record(stream)
                fn()
                b.record(stream)
            torch.cuda.synchronize()
            tot += a.elapsed_time(b)
        return tot / args.iters

    with torch.cuda.stream(stream):
        h1 = cf.from_synth(m, stream=stream)
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    ins1 = (t(s.x), t(s.v), t(s.e), t(s.rho0detJ0))
    out1 = h1.alloc_outputs()
    t1 = time_fn(lambda: h1.eval(*ins1, out=out1))
    h1.set_timing(True)
    h1.eval(*ins1, out=out1)
    torch.cuda.synchronize()
    k1 = h1.kernel_times()
    h1.set_timing(False)
    res = {"config": args.config, "zones": m.num_zones, "t1_ms": t1, "t1_kb1_ms": k1[0], "t1_kb2_ms": k1[1],
           "variant": h1.variant, "l2": "flushed before every timed eval", "ranks": []}
    h1.close()
    for P in [int(p) for p in args.ranks.split(",")]:
        if P == 1:
            continue
        parts = synth.partition(m, P)
        per = []
        for r, p in enumerate(parts):
            lm, ls = p.local_mesh(m), p.local_state(s)
            with torch.cuda.stream(stream):
                h = cf.from_synth(lm, params=par, stream=stream)
            ins = (t(ls.x), t(ls.v), t(ls.e), t(ls.rho0detJ0))
            out = h.alloc_outputs()
            tr = time_fn(lambda: h.eval(*ins, out=out))
            h.set_timing(True)
            h.eval(*ins, out=out)
            torch.cuda.synchronize()
            kt = h.kernel_times()
            h.set_timing(False)
            per.append({"rank": r, "zones": lm.num_zones, "nodes": lm.num_nodes, "ms": tr, "kb1_ms": kt[0],
                        "kb2_ms": kt[1]})
            h.close()
        tmax = max(q["ms"] for q in per)
        with torch.cuda.stream(stream):   # the overlap schedule each rank would run (no NCCL call is made)
            hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None, stream=stream) for p in parts]
        modes = [h.exchange_schedule() for h in hs]
        for h in hs:
            h.close()
        shared = [int(p.nbr_offset[-1]) for p in parts]
        res["ranks"].append({"P": P, "max_rank_ms": tmax, "E_compute": t1 / (P * tmax),
                             "per_rank": per, "schedule": [{"mode": md, "boundary_zones": nb} for md, nb in modes],
                             "shared_rows_per_rank": shared, "message_bytes_per_rank": [r_ * m.dim * 8 for r_ in shared]})
        print(f"P={P}: max rank {tmax:.4f} ms (t1 {t1:.4f}) E_compute {t1 / (P * tmax):.3f}", file=sys.stderr)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
