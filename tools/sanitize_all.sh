#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck / initcheck over the cases of tools/sanitize.py (under gpurun)
mkdir -p gpurun_out
out=gpurun_out/r02s3_sanitizer.txt
: > $out
for tool in memcheck synccheck racecheck initcheck; do
  for c in c4 c5 c5v8 c3 c2 integrator host loopback; do
    if { [ $tool = racecheck ] || [ $tool = initcheck ]; } && { [ $c = host ] || [ $c = loopback ]; }; then continue; fi
    echo "=== $tool $c" >> $out
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py $c >> $out 2>&1
    echo "rc=$?" >> $out
  done
done
grep -E "^===|ERROR SUMMARY|RACECHECK SUMMARY|rc=" $out
