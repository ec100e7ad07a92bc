timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t4.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t4.log
tail -15 gpurun_out/t4.log
for c in C4 C3 C5 C2; do timeout 300 python bench.py --config $c --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench4_$c.log 2>&1; tail -1 gpurun_out/bench4_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'][:40], d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_v3 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full4.log 2>&1
tail -2 gpurun_out/ncu_full4.log
