"""How often the dt filter's exact sigma_min(J) runs (v10 DIAG 4 counters, diagnostics build):
BLAST_CF_PROFILE=1 BLAST_CF_KB1=v10.wpxd4 python tools/dt_exact_rate.py [C4] [S1]"""
import os, sys
os.environ["BLAST_CF_PROFILE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_dongdkrtd14_b200 as cf, synth
cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
m, s = synth.config(cfg, sys.argv[2] if len(sys.argv) > 2 else "S1")
h = cf.from_synth(m)
t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
h.eval(x, v, e, r)
torch.cuda.synchronize()
st = h.debug_stage_clocks().astype(float)
nv, nx = st[:, 12].sum(), st[:, 13].sum()
print(f"{cfg} {h.variant}: warp votes {nv:.0f}, exact dt evaluated {nx:.0f} ({100 * nx / max(nv, 1):.1f} %)")
