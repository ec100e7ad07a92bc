#!/bin/bash
# usage (under gpurun): tools/bench_variants.sh <tag> <config> <variant> [<variant> ...]
# one device-timed bench line per KB1 variant (BLAST_CF_KB1), summarised as: variant ms/step KB1 ms frac
tag=$1; cfg=$2; shift 2
mkdir -p gpurun_out
for V in "$@"; do
  BLAST_CF_KB1=$V timeout 300 python bench.py --config $cfg --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-energy \
    > gpurun_out/${tag}_$V.jsonl 2> gpurun_out/${tag}_$V.err
  python - "$V" "gpurun_out/${tag}_$V.jsonl" <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); r = d["roofline"]
    print(f"{sys.argv[1]:10s} step {d['ms_per_step']:.4f} ms  KB1 {r['kernel_ms']:.4f} ms  frac {r['frac']:.3f}  clocks {d['clocks']['sm_mhz']}  regs {d['launch']['regs_per_thread']} local {d['launch']['local_bytes']}")
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
