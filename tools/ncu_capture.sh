#!/bin/bash
# usage (under gpurun): tools/ncu_capture.sh <tag> <config> <kernel-regex> [extra env]
# one ncu --set full capture (with source) of the top kernel of a short bench run; the report lands in gpurun_out/
tag=$1; cfg=$2; rx=$3
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$rx" -s 2 -c 1 -f -o gpurun_out/$tag \
  python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-energy > gpurun_out/$tag.log 2>&1
echo "ncu $tag rc=$?"
