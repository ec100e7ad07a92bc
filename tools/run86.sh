# final validation after the p2d / v2.z1m12 defaults
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t86.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t86.log; tail -3 gpurun_out/t86.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke86.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke86.log
summ() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); r=d['roofline']; print('$1', '%.4e'%d['value'], round(d['ms_per_step'],4), round(r['frac'],4), round(r['kernel_ms'],4), r['kernel'], '%.3e'%d['e2e']['value'], r['traffic'])"; }
timeout 400 python bench.py > gpurun_out/b86_C4.log 2>&1; summ gpurun_out/b86_C4.log
for C in C2 C3 C5; do timeout 400 python bench.py --config $C > gpurun_out/b86_$C.log 2>&1; summ gpurun_out/b86_$C.log; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/b86_ref.log 2>&1; tail -c 200 gpurun_out/b86_ref.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_C2_r86 python bench.py --config C2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu86.log 2>&1; tail -1 gpurun_out/ncu86.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c4_r86.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncul86.log 2>&1
