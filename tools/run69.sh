mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "variant" > gpurun_out/t69.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t69.log; tail -3 gpurun_out/t69.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'])"; }
for V in v10.w v10.v v10.wr3; do BLAST_CF_KB1=$V timeout 300 python bench.py --config C4 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b69_$V.log 2>&1; summ gpurun_out/b69_$V.log; done
for V in v10.wd1 v10.w; do echo -n "$V "; BLAST_CF_KB1=$V timeout 120 python tools/kw_stages.py C4; done
