timeout 600 python -m pytest tests -m gpu -x -q -k "3d_all or configs_small or full_size or loopback or variant" > gpurun_out/t22.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t22.log
tail -3 gpurun_out/t22.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'], d.get('energy'))"; }
timeout 200 python bench.py --config C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b22_c5.log 2>&1; summ gpurun_out/b22_c5.log
BLAST_CF_KB1=v1.z1 timeout 200 python bench.py --config C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b22_c5b.log 2>&1; summ gpurun_out/b22_c5b.log
timeout 200 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b22_c4.log 2>&1; summ gpurun_out/b22_c4.log
