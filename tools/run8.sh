timeout 300 python tools/stage_profile.py C4 load,A,B,C+pw,SBwrite,CT,BT,AT+dt
timeout 300 python tools/stage_profile.py C3 load,A,B,C+pw,SBwrite,CT,BT,AT+dt
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
timeout 300 python bench.py --config C4 --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b8_c4.log 2>&1; summ gpurun_out/b8_c4.log
timeout 600 python -m pytest tests -m gpu -x -q -k "configs_small or determinism or full_size" 2>&1 | tail -2
