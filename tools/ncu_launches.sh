#!/bin/bash
# ncu launch list (gpu__time_duration per launch, cold / serialised) of a short bench run: profiles' kernel shares
cfg=$1; out=gpurun_out/r02s3_launches_$cfg.csv
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $out \
  python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-energy > /dev/null 2>&1
echo "launches $cfg rc=$?"
