timeout 600 python bench.py --steps 200 --warmup 5 --cpu-seconds 20 > gpurun_out/bench17.log 2>&1; tail -1 gpurun_out/bench17.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 --cpu-seconds 30 > gpurun_out/bench17_ref.log 2>&1; tail -1 gpurun_out/bench17_ref.log
