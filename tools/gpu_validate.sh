set -x
mkdir -p gpurun_out
nvidia-smi -L
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_pytest.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed|FAILED|Error" gpurun_out/r2_pytest.log | tail -40
timeout 300 python bench.py --config C4 --steps 20 --warmup 3 > gpurun_out/r2_bench_c4.jsonl 2> gpurun_out/r2_bench_c4.err; echo "bench rc=$?"
tail -c 3000 gpurun_out/r2_bench_c4.jsonl
