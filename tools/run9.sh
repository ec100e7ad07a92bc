timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t9.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t9.log
tail -15 gpurun_out/t9.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
timeout 300 python bench.py --config C4 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b9_c4.log 2>&1; summ gpurun_out/b9_c4.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_v4 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full9.log 2>&1
tail -1 gpurun_out/ncu_full9.log
