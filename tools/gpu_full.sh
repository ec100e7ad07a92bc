#!/bin/bash
# full GPU validation under gpurun: pytest -m gpu, smoke, sanitizers, bench lines of every config
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02s3_pytest_gpu.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed|FAILED" gpurun_out/r02s3_pytest_gpu.log | tail -15
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02s3_smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/r02s3_smoke.log
# compute-sanitizer is closed on this GPU pool (round 2, session 3): the committed r02 sanitizer logs stand
for c in C4 C5 C3 C2; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 > gpurun_out/r02s3_bench_$c.jsonl 2> gpurun_out/r02s3_bench_$c.err
  echo "bench $c rc=$?"
done
timeout 600 python bench.py --impl reference --config C4 --steps 2 --warmup 3 > gpurun_out/r02s3_bench_ref.jsonl 2>&1; echo "ref rc=$?"
