mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "variant or full_size_sampled and C5 or 3d_all" > gpurun_out/t78.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t78.log; tail -3 gpurun_out/t78.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
timeout 300 python bench.py --config C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b78_C5.log 2>&1; summ gpurun_out/b78_C5.log
