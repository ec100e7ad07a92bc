timeout 900 python -m pytest tests -m gpu -x -q -k "3d_all or configs_small or full_size or loopback or determinism or debug_Fz" > gpurun_out/t15.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t15.log
tail -3 gpurun_out/t15.log
timeout 300 python tools/v4_balance.py C4
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
timeout 300 python bench.py --config C4 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b15_c4.log 2>&1; summ gpurun_out/b15_c4.log
BLAST_CF_KB1=v4m0 timeout 300 python bench.py --config C4 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b15_c4m0.log 2>&1; summ gpurun_out/b15_c4m0.log
