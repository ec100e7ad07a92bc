mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "variant or full_size_sampled or configs_small or 3d_all" > gpurun_out/t82.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t82.log; tail -3 gpurun_out/t82.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'], r['traffic'])"; }
timeout 400 python bench.py --config C3 > gpurun_out/b82_C3.log 2>&1; summ gpurun_out/b82_C3.log
for C in C3 C2; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_${C}_r82 python bench.py --config $C --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu82_$C.log 2>&1; tail -1 gpurun_out/ncu82_$C.log; done
