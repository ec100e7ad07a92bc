timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > gpurun_out/t3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t3.log
tail -15 gpurun_out/t3.log
timeout 300 python bench.py --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench3.log 2>&1; tail -1 gpurun_out/bench3.log | cut -c1-1500
BLAST_CF_KB1=v1 timeout 300 python bench.py --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench3v1.log 2>&1; tail -1 gpurun_out/bench3v1.log | cut -c1-600
timeout 300 python bench.py --config C3 --steps 100 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench3c3.log 2>&1; tail -1 gpurun_out/bench3c3.log | cut -c1-600
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_v2 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full3.log 2>&1
tail -2 gpurun_out/ncu_full3.log
