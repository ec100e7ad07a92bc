mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "variant or full_size or 2d or 3d_all" > gpurun_out/t70.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t70.log; tail -3 gpurun_out/t70.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
for C in C4 C3 C5 C2; do timeout 300 python bench.py --config $C --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b70_$C.log 2>&1; summ gpurun_out/b70_$C.log; done
