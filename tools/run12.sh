timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t12.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t12.log
tail -15 gpurun_out/t12.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_c4_v4b python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full12.log 2>&1
tail -1 gpurun_out/ncu_full12.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_c4_v4.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch12.log 2>&1
tail -1 gpurun_out/ncu_launch12.log
