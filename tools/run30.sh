timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t30.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t30.log
tail -3 gpurun_out/t30.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke30.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke30.log; tail -3 gpurun_out/smoke30.log
timeout 400 python bench.py > gpurun_out/b30.log 2>&1; tail -1 gpurun_out/b30.log
