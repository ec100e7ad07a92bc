mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "2d" > gpurun_out/t85.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t85.log; tail -3 gpurun_out/t85.log
python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_ipps_dongdkrtd14_b200 as cf
mesh, st = synth.config("C2", "S1")
h = cf.from_synth(mesh)
print("C2", h.autotune(*[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in (st.x, st.v, st.e, st.rho0detJ0)], reps=50), flush=True)
PY
