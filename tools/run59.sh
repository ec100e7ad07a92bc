# v10 default: full GPU suite, C4 bench line, v10.q timing, ncu full capture + launch list of the default
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t59.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t59.log; tail -3 gpurun_out/t59.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
timeout 400 python bench.py > gpurun_out/b59_C4.log 2>&1; summ gpurun_out/b59_C4.log
BLAST_CF_KB1=v10.q timeout 300 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b59_v10q.log 2>&1; summ gpurun_out/b59_v10q.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_C4_v10 python bench.py --config C4 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu59.log 2>&1; tail -1 gpurun_out/ncu59.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c4_v10.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncul59.log 2>&1
