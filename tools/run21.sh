./tools/mufu_accuracy
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/t21.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t21.log
tail -3 gpurun_out/t21.log
