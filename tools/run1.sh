set -x
nvidia-smi -L
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > gpurun_out/t1.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t1.log
tail -30 gpurun_out/t1.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; tail -5 gpurun_out/smoke.log
timeout 600 python bench.py --steps 10 --warmup 3 --cpu-seconds 5 > gpurun_out/bench1.log 2>&1; tail -3 gpurun_out/bench1.log
