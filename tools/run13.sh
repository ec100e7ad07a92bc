timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t13.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t13.log
tail -4 gpurun_out/t13.log
timeout 300 python tools/v4_balance.py C4
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
for c in C4 C3 C5 C2; do timeout 300 python bench.py --config $c --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b13_$c.log 2>&1; summ gpurun_out/b13_$c.log; done
