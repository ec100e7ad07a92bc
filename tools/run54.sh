# pipelined eval_host: bitwise tests, then the e2e of every config
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_host or variant" > gpurun_out/t54.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t54.log; tail -3 gpurun_out/t54.log
for C in C4 C3 C5 C2; do
timeout 400 python bench.py --config $C --steps 50 --warmup 3 --no-cpu-baseline > gpurun_out/b54_$C.log 2>&1
python -c "import json; d=json.loads(open('gpurun_out/b54_$C.log').read().strip().splitlines()[-1]); print('$C', '%.4e'%d['value'], '%.4e'%d['e2e']['value'], round(d['e2e']['ms_per_step'],3), round(d['ms_per_step'],4))"
done
