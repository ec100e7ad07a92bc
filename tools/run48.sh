timeout 900 python -m pytest tests -m gpu -x -q -k "variant" > gpurun_out/t48.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t48.log; tail -3 gpurun_out/t48.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['launch'])"; }
for V in v8 v8.m1 v1.z1m2; do
BLAST_CF_KB1=$V timeout 300 python bench.py --config C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b48_$V.log 2>&1; summ gpurun_out/b48_$V.log
done
