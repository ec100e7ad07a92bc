timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/t23.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t23.log
tail -3 gpurun_out/t23.log
timeout 120 python tools/v4_balance.py C4
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
timeout 120 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b23_c4.log 2>&1; summ gpurun_out/b23_c4.log
timeout 120 python bench.py --config C4 --state S0 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b23_c4s0.log 2>&1; summ gpurun_out/b23_c4s0.log
