import os, sys
os.environ["BLAST_CF_PROFILE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_dongdkrtd14_b200 as cf, synth
m, s = synth.config(sys.argv[1] if len(sys.argv) > 1 else "C4", "S1")
h = cf.from_synth(m)
t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
for _ in range(3): h.eval(x, v, e, r)
torch.cuda.synchronize()
st = h.debug_stage_clocks().astype(float)
print("PW busy", np.median(st[:, 0]), "KW busy", np.median(st[:, 1]), "loop", np.median(st[:, 2]))
print("zones/CTA", m.num_zones / len(st), "cycles per zone: PW", np.median(st[:, 0]) / (m.num_zones / len(st)),
      "KW", np.median(st[:, 1]) / (m.num_zones / len(st)), "loop", np.median(st[:, 2]) / (m.num_zones / len(st)))
