timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t46.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t46.log; tail -2 gpurun_out/t46.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke46.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke46.log; tail -3 gpurun_out/smoke46.log
timeout 400 python bench.py > gpurun_out/b46.log 2>&1; tail -1 gpurun_out/b46.log
timeout 400 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/b46ref.log 2>&1; tail -1 gpurun_out/b46ref.log
