# PW-alone / KW-alone stage clocks of v5, v6, v10 (same build), C4
for V in v5.d1 v6.d1 v10.d1 v5.r1d1 v5.d2 v10.d2 v10 v5.r1; do echo -n "$V "; BLAST_CF_KB1=$V timeout 120 python tools/kw_stages.py C4; done
