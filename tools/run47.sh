timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c5 python bench.py --config C5 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu47.log 2>&1
tail -1 gpurun_out/ncu47.log
