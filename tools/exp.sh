#!/bin/bash
# usage: tools/exp.sh <tag> <config> <pytest -k expr or ""> <variant>...   (diagnostics build here, then one gpurun call:
# the variant parity tests selected by -k, then one bench line per variant)
tag=$1; cfg=$2; kx=$3; shift 3
BLAST_CF_NVCC_FLAGS=-DBLAST_CF_DIAGNOSTICS python -c "from paper_conf_ipps_dongdkrtd14_b200 import build; build.build(force=True)" > /tmp/exp_build.log 2>&1 || { grep -i error /tmp/exp_build.log | head; exit 1; }
cmd=""
[ -n "$kx" ] && cmd="python -m pytest tests/test_gpu_parity.py -q -x -k \"$kx\" -p no:cacheprovider 2>&1 | tail -3; "
cmd="$cmd bash tools/bench_variants.sh $tag $cfg $*"
/usr/local/graft/bin/gpurun --timeout 900 -- "$cmd" > gpurun_out/call_$tag.log 2>&1
grep -v '^\[gpurun\] merged\|^\[gpurun\] sending' gpurun_out/call_$tag.log | tail -14
