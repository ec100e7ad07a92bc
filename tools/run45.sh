summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['config']['workload'], d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'].get('regs_per_thread'))"; }
for C in C2 C3 C5; do
timeout 200 python bench.py --config $C --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b45_$C.log 2>&1; summ gpurun_out/b45_$C.log
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_r45.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu45a.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_v5r1 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu45b.log 2>&1
tail -1 gpurun_out/ncu45b.log
