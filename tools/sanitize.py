#!/usr/bin/env python
"""One small corner-force evaluation (or integrator step) for compute-sanitizer.

    compute-sanitizer --tool memcheck|racecheck|synccheck python tools/sanitize.py <case>
cases: c4 (v10.wpx, 3D k=4, 40 zones), c5 (v11.mbtsiet, 3D k=8, 4 zones), c5v8 (v8), c3 (v2.z1m12e, 3D k=2),
       c2 (p2d.z2m6, 2D k=4), integrator (2D k=3 RK2 step), host (pipelined host entry, 3D k=2 16^3),
       loopback (the overlap schedule of a 4-rank loopback group), p2p (2 processes, the peer-memory exchange
       over CUDA IPC, 3 evals each; compute-sanitizer follows the child processes)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
CASES = {"c4": ("C4", (5, 4, 2), None, "v10.wpx"), "c5": ("C5", (2, 1, 2), None, "v11.mbtsiet"), "c5v8": ("C5", (2, 1, 2), None, "v8"),
         "c3": ("C3", (4, 4, 3), None, "v2.z1m12e"), "c2": ("C2", (9, 7), None, "p2d.z2m6")}


def _p2p_rank(rank, world, port):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    m, s = synth.config("C3", "S1", N=(6, 4, 4))
    par = cf.default_params()
    par.h0 = (1.0 / m.num_zones) ** (1 / 3) / m.order
    p = synth.partition(m, world)[rank]
    h = cf.from_synth(m, params=par, part=p, nccl_uid=None)
    h.p2p_connect()
    ls = p.local_state(s)
    for _ in range(3):
        o = h.eval(t(ls.x), t(ls.v), t(ls.e), t(ls.rho0detJ0))
    torch.cuda.synchronize()
    print("p2p rank", rank, h.exchange_schedule(), float(o[2].cpu()[0]))
    h.close()
    dist.destroy_process_group()


def main(case):
    import torch
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    if case in CASES:
        name, N, k, var = CASES[case]
        os.environ["BLAST_CF_KB1"] = var
        m, s = synth.config(name, "S1", N=N, k=k)
        h = cf.from_synth(m)
        assert h.variant == var, h.variant
        for _ in range(2):
            F1, FTv, dt = h.eval(t(s.x), t(s.v), t(s.e), t(s.rho0detJ0))
        torch.cuda.synchronize()
        print(case, var, "dt", float(dt.cpu()[0]), "|F1|", float(F1.abs().max()))
    elif case == "integrator":
        m = synth.make_mesh("triple", 2, 3, (7, 3))
        s = synth.make_state(m, "triple", "S1", 1)
        h = cf.from_synth(m)
        rk = cf.RK2(h, s.rho0detJ0)
        x, v, e = t(s.x), t(s.v), t(s.e)
        d, it = rk.step(x, v, e, 1e-3)
        torch.cuda.synchronize()
        print(case, "dt_est", d, "cg", it)
    elif case == "host":
        m, s = synth.config("C3", "S1", N=(16, 16, 16))
        h = cf.from_synth(m)
        hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (s.x, s.v, s.e, s.rho0detJ0)]
        o = h.eval_host(*hx)
        h.set_rho0detJ0_host(hx[3])
        o = h.eval_host(hx[0], hx[1], hx[2], None)
        print(case, "dt", o[2][0])
    elif case == "p2p":
        import socket
        import torch.multiprocessing as mp
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        mp.spawn(_p2p_rank, args=(2, port), nprocs=2, join=True)
        print(case, "ok")
    elif case == "loopback":   # the overlap schedule of the multi-rank exchange (comm streams, events)
        m, s = synth.config("C3", "S1", N=(8, 6, 6))
        par = cf.default_params()
        par.h0 = (1.0 / m.num_zones) ** (1 / 3) / m.order
        parts = synth.partition(m, 4)
        hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None) for p in parts]
        ls = [p.local_state(s) for p in parts]
        outs = cf.eval_loopback(hs, [t(l.x) for l in ls], [t(l.v) for l in ls], [t(l.e) for l in ls],
                                [t(l.rho0detJ0) for l in ls])
        torch.cuda.synchronize()
        print(case, [h.exchange_schedule() for h in hs], float(outs[0][2].cpu()[0]))
    else:
        raise SystemExit(f"unknown case {case}")
    return 0


if __name__ == "__main__":
    sys.exit(main(sys.argv[1]))
