summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
BLAST_CF_KB1=v4m1 timeout 120 python bench.py --config C4 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b16_c4m1.log 2>&1; summ gpurun_out/b16_c4m1.log
BLAST_CF_KB1=v4m1 timeout 300 python -m pytest tests -m gpu -x -q -k "3d_all_orders or configs_small or full_size" 2>&1 | tail -2
