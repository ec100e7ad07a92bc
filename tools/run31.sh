timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_r31 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu31.log 2>&1
tail -2 gpurun_out/ncu31.log
ls -la gpurun_out
