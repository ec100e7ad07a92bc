summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', round(d['ms_per_step'],4), round(r['kernel_ms'],4), r['kernel'])"; }
mkdir -p gpurun_out
for V in v10.wq v10.wl v10.w; do BLAST_CF_KB1=$V timeout 200 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b89_$V.log 2>&1; summ gpurun_out/b89_$V.log; done
