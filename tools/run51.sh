# dt filter in v2/v3, rho0|J0| L1 prefetch in v3/v8: GPU tests + C3/C5/C2 bench lines
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t51.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t51.log; tail -3 gpurun_out/t51.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
for C in C3 C5 C2; do
timeout 300 python bench.py --config $C --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b51_$C.log 2>&1; summ gpurun_out/b51_$C.log
done
for V in v3.z2 v2.z2; do
BLAST_CF_KB1=$V timeout 300 python bench.py --config C3 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
done
python - <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, '.')
import synth, paper_conf_ipps_dongdkrtd14_b200 as cf
for k in (3,):
    mesh, st = synth.config("C3", "S1", k=k)
    h = cf.from_synth(mesh)
    print(k, h.autotune(*[torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in (st.x, st.v, st.e, st.rho0detJ0)], reps=20))
PY
