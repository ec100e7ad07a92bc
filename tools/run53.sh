# v2 one-point-per-thread variants: parity + autotune timings on C3 (k=2) and 32^3 k=3, k=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "variant" > gpurun_out/t53.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t53.log; tail -3 gpurun_out/t53.log
python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_ipps_dongdkrtd14_b200 as cf
for k in (2, 3, 1):
    mesh, st = synth.config("C3", "S1", k=k)
    h = cf.from_synth(mesh)
    print(k, h.autotune(*[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in (st.x, st.v, st.e, st.rho0detJ0)], reps=20), flush=True)
PY
