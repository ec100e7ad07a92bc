#!/usr/bin/env python
"""The paper's validation run (Table 6): 2D triple point, Q3-Q2, to t = 0.6, on the GPU.

Reports the kinetic / internal / total discrete energies at t = 0 and t = 0.6 and the total-energy change
(Table 6: total ~10.05, change -9.22e-13 (CPU) / -4.94e-13 (GPU)).  The mesh resolution is not printed in
the paper; 56 x 24 zones is the 7:3-aligned mesh on which the initial condition of reading R17 gives
IE0 = 201/20 = 10.05 exactly (tests/test_generator.py).  Integrator: the library's RK2-average step with the
R24 step control and CG tolerance 1e-14 (blast_cf_rk2_advance).  One JSON line on stdout.

    python tools/table6.py [--N 56 24] [--t-final 0.6] [--out profiles/r02_table6.json]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, nargs=2, default=[56, 24])
    ap.add_argument("--k", type=int, default=3)
    ap.add_argument("--t-final", type=float, default=0.6)
    ap.add_argument("--max-steps", type=int, default=100000)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    m = synth.make_mesh("triple", 2, a.k, tuple(a.N))
    s = synth.make_state(m, "triple", "S0", 1)
    h = cf.from_synth(m)
    rk = cf.RK2(h, s.rho0detJ0, cg_rel_tol=1e-14)
    t = lambda arr: torch.from_numpy(np.ascontiguousarray(arr)).cuda()
    x, v, e = t(s.x), t(s.v), t(s.e)
    ke0, ie0 = rk.energy(v, e)
    _, _, dt0 = h.eval(x, v, e, t(s.rho0detJ0))
    dt = 0.5 * float(dt0.cpu()[0])
    torch.cuda.synchronize()
    w0 = time.perf_counter()
    tr, dtn, steps, rej = rk.advance(x, v, e, a.t_final, dt, a.max_steps)
    torch.cuda.synchronize()
    wall = time.perf_counter() - w0
    ke, ie = rk.energy(v, e)
    E0, E1 = ke0 + ie0, ke + ie
    line = {"run": "Table 6 (PAPER.md:894-900): 2D triple point Q%d-Q%d, %dx%d zones" % (a.k, a.k - 1, *a.N),
            "t_reached": tr, "steps": steps, "rejected": rej, "wall_s": wall,
            "t0": {"kinetic": ke0, "internal": ie0, "total": E0},
            "t_final": {"kinetic": ke, "internal": ie, "total": E1},
            "delta_total": E1 - E0, "rel_delta_total": (E1 - E0) / E0,
            "paper": {"total": 10.05, "delta_cpu": -9.22e-13, "delta_gpu": -4.94e-13},
            "min_x_change": float((x - t(s.x)).abs().max().cpu())}
    print(json.dumps(line))
    if a.out:
        with open(a.out, "w") as f:
            json.dump(line, f, indent=1)
    return 0


if __name__ == "__main__":
    sys.exit(main())
