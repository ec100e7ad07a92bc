"""Per-stage cycle split of the contraction warps of kb1_v6 (BLAST_CF_PROFILE=1 stage clocks).
usage: BLAST_CF_KB1=v6[.d2] python tools/kw_stages.py [C4]"""
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
zpc = m.num_zones / len(st)
names = {0: "PW busy", 1: "KW busy", 2: "PW loop", 3: "issue", 4: "C^T", 5: "B^T", 6: "A^T", 7: "cp.wait+bar",
         8: "fwd A", 9: "fwd B", 10: "fwd C_x", 11: "CTA bar"}
print(" ".join(f"{names[k]}={np.median(st[:, k]) / zpc:.0f}" for k in range(12)))
