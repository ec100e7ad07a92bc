# f2: multi-rank CG (loopback group) + integrator regression
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_integrator.py -x -q > gpurun_out/t60.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t60.log; tail -30 gpurun_out/t60.log
