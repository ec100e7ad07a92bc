python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_ipps_dongdkrtd14_b200 as cf
mesh, st = synth.config("C2", "S1")
h = cf.from_synth(mesh)
print("C2", h.autotune(*[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in (st.x, st.v, st.e, st.rho0detJ0)], reps=50), flush=True)
PY
