"""KB1's fixed per-launch cost: KB1 time on C4-recipe meshes of m zones per CTA (148 CTAs), fit t = a + b m.
python tools/fixed_cost.py   (one GPU; BLAST_CF_KB1 picks the variant)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_dongdkrtd14_b200 as cf, synth
res = []
for N in [(37, 4, 1), (37, 4, 2), (37, 4, 4), (37, 8, 4), (37, 8, 8), (37, 16, 8), (74, 16, 8)]:
    m, s = synth.config("C4", "S1", N=N)
    h = cf.from_synth(m)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
    h.set_timing(True)
    for _ in range(3): h.eval(x, v, e, r)
    ts = []
    for _ in range(20):
        h.eval(x, v, e, r); torch.cuda.synchronize(); ts.append(h.kernel_times()[0])
    zpc = m.num_zones / 148
    res.append((zpc, float(np.median(ts))))
    print(f"{h.variant} zones {m.num_zones} per CTA {zpc:.1f}: KB1 {np.median(ts) * 1e3:.2f} us", flush=True)
    h.close()
z, tt = np.array(res).T
b, a = np.polyfit(z, tt, 1)
print(f"fit: KB1 = {a * 1e3:.1f} us + {b * 1e3:.3f} us per zone per CTA")
