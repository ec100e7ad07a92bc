# session 3 first call: full GPU tests, bench lines of every config, ncu captures of KB1 for C2/C3/C5 (traffic)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t50.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t50.log; tail -3 gpurun_out/t50.log
for C in C4 C2 C3 C5; do
timeout 400 python bench.py --config $C > gpurun_out/b50_$C.log 2>&1; tail -c 600 gpurun_out/b50_$C.log; echo
done
for C in C2 C3 C5; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kb1 -s 3 -c 1 -o gpurun_out/kb1_${C}_r50 python bench.py --config $C --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu50_$C.log 2>&1
tail -1 gpurun_out/ncu50_$C.log
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c4_r50.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncul50.log 2>&1
