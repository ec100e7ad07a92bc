mkdir -p gpurun_out
BLAST_CF_KB1=v10.w timeout 120 python -c "
import sys; sys.path.insert(0,'.')
import numpy as np, torch, synth, paper_conf_ipps_dongdkrtd14_b200 as cf
m,s=synth.config('C4','S1',N=(5,3,2)); h=cf.from_synth(m); t=lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
o=h.eval(t(s.x),t(s.v),t(s.e),t(s.rho0detJ0)); torch.cuda.synchronize(); print('small ok', h.variant)
m,s=synth.config('C4','S1'); h=cf.from_synth(m)
o=h.eval(t(s.x),t(s.v),t(s.e),t(s.rho0detJ0)); torch.cuda.synchronize(); print('full ok', h.variant)
" > gpurun_out/x74.log 2>&1; echo "probe rc=$?"; tail -3 gpurun_out/x74.log
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "variant" > gpurun_out/t74.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t74.log; tail -3 gpurun_out/t74.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
for V in v10.w; do BLAST_CF_KB1=$V timeout 200 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b74_$V.log 2>&1; summ gpurun_out/b74_$V.log; done
for V in v10.w; do echo -n "$V "; BLAST_CF_KB1=$V timeout 120 python tools/kw_stages.py C4; done
