#!/bin/bash
# C5 v11 default validation (under gpurun): parity, sanitizers, ncu capture, launch list
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider 2>&1 | tail -3
out=gpurun_out/r02_sanitizer_c5_mbtsi.txt; : > $out
for tool in memcheck synccheck racecheck initcheck; do
  echo "=== $tool c5" >> $out
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py c5 >> $out 2>&1
  echo "rc=$?" >> $out
done
grep -E "^===|ERROR SUMMARY|RACECHECK SUMMARY|rc=" $out
bash tools/ncu_capture.sh c5_v11mbtsi C5 kb1_v11
bash tools/ncu_launches.sh C5
