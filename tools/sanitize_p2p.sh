mkdir -p gpurun_out
out=gpurun_out/r02_sanitizer_p2p.txt; : > $out
for tool in memcheck synccheck initcheck; do
  echo "=== $tool p2p" >> $out
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py p2p >> $out 2>&1
  echo "rc=$?" >> $out
done
grep -E "^===|ERROR SUMMARY|rc=|p2p rank" $out
timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_multirank.py -q -p no:cacheprovider 2>&1 | tail -3
