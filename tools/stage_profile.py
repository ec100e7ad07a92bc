"""Per-stage cycle breakdown of KB1 from the clock64 stamps (BLAST_CF_PROFILE=1)."""
import os
import sys

os.environ["BLAST_CF_PROFILE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ipps_dongdkrtd14_b200 as cf
import synth

name = sys.argv[1] if len(sys.argv) > 1 else "C4"
names = sys.argv[2].split(",") if len(sys.argv) > 2 else None
m, s = synth.config(name, "S1")
h = cf.from_synth(m)
t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
for _ in range(3):
    h.eval(x, v, e, r)
torch.cuda.synchronize()
st = h.debug_stage_clocks()
ns = int((st != 0).sum(1).max())
d = np.diff(st[:, :ns], axis=1).astype(np.float64)
tot = (st[:, ns - 1] - st[:, 0]).astype(np.float64)
print(f"{name}: CTAs {len(st)}, stamps {ns}, median CTA cycles {np.median(tot):.0f}")
for i in range(ns - 1):
    lab = names[i] if names and i < len(names) else f"seg{i}"
    print(f"  {lab:12s} median {np.median(d[:, i]):8.0f} cyc  mean {d[:, i].mean():8.0f}  share {d[:, i].sum() / tot.sum():.3f}")
