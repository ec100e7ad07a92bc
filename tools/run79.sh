mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t79.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t79.log; tail -3 gpurun_out/t79.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke79.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke79.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'], '%.3e'%d['e2e']['value'], r['traffic'])"; }
timeout 400 python bench.py > gpurun_out/b79_C4.log 2>&1; summ gpurun_out/b79_C4.log
for C in C2 C3 C5; do timeout 400 python bench.py --config $C > gpurun_out/b79_$C.log 2>&1; summ gpurun_out/b79_$C.log; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/b79_ref.log 2>&1; tail -c 400 gpurun_out/b79_ref.log
