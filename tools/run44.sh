summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], round(d['roofline']['frac'],4), d['roofline']['kernel_ms'], d['roofline']['kb2_ms'], d['launch'])"; }
for V in v4.m0 v5.r1 v5 v4.m0 v5.r1; do
BLAST_CF_KB1=$V timeout 120 python bench.py --config C4 --steps 200 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b44_$V.log 2>&1; summ gpurun_out/b44_$V.log
done
timeout 300 python -m pytest tests -m gpu -x -q -k "variant or autotune" 2>&1 | tail -1
