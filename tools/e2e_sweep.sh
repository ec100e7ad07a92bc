for cfg in C3 C4; do for set in "8 0" "6 1.5" "8 1.5" "4 1.5"; do set -- $set; for rep in 1 2; do
  BLAST_CF_HOST_CHUNKS=$1 BLAST_CF_HOST_TAPER=$2 timeout 300 python bench.py --config $cfg --steps 10 --warmup 3 --no-cpu-baseline --no-energy 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$cfg chunks $1 taper $2', round(d['e2e']['ms_per_step'],3))"
done; done; done
