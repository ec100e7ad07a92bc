#!/usr/bin/env python
"""e2e diagnostic: pinned H2D / D2H bandwidth for the C4 per-step volumes, and the host-entry time."""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    dev = torch.device("cuda", 0)
    for mb in (16, 120, 256):
        n = mb * 2 ** 20 // 8
        h = torch.empty(n, dtype=torch.float64).pin_memory()
        d = torch.empty(n, dtype=torch.float64, device=dev)
        s = torch.cuda.Stream()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            for _ in range(2):
                d.copy_(h, non_blocking=True)
            e0.record(s)
            for _ in range(5):
                d.copy_(h, non_blocking=True)
            e1.record(s)
        torch.cuda.synchronize()
        h2d = 5 * n * 8 / (e0.elapsed_time(e1) / 1e3) / 1e9
        with torch.cuda.stream(s):
            e0.record(s)
            for _ in range(5):
                h.copy_(d, non_blocking=True)
            e1.record(s)
        torch.cuda.synchronize()
        d2h = 5 * n * 8 / (e0.elapsed_time(e1) / 1e3) / 1e9
        print(f"{mb} MB: H2D {h2d:.1f} GB/s  D2H {d2h:.1f} GB/s")
    m, st = synth.config("C4", "S1")
    h = cf.from_synth(m)
    hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (st.x, st.v, st.e, st.rho0detJ0)]
    h.set_rho0detJ0_host(hx[3])
    out = (torch.empty(tuple((3, m.num_nodes)), dtype=torch.float64).pin_memory(),
           torch.empty(tuple((m.num_zones, m.nt)), dtype=torch.float64).pin_memory(),
           torch.empty(1, dtype=torch.float64).pin_memory())
    for _ in range(3):
        h.eval_host(hx[0], hx[1], hx[2], None, out=out)
    t0 = time.perf_counter()
    for _ in range(10):
        h.eval_host(hx[0], hx[1], hx[2], None, out=out)
    print("eval_host C4: %.3f ms (wall)" % ((time.perf_counter() - t0) / 10 * 1e3))


if __name__ == "__main__":
    main()
