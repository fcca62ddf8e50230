#!/bin/bash
# Decode attention source-level ncu (arXiv mix, 70 SMs): per-SASS stall samples.
set -u
O=gpurun_out/${OUT:-s12}; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
timeout 600 $F -k regex:k_attn_decode -s 1 -c 1 -o $O/attn_dec_p78 python scripts/prof_step.py --reps 2 --quiet --mode dec --p 78 --config arxiv-8b > $O/ncu.log 2>&1
ncu -i $O/attn_dec_p78.ncu-rep --page source --csv --print-source sass > $O/attn_dec_p78.sass.csv 2>/dev/null
ncu -i $O/attn_dec_p78.ncu-rep --page source --csv --print-source cuda > $O/attn_dec_p78.cuda.csv 2>/dev/null
ncu -i $O/attn_dec_p78.ncu-rep --page raw --csv > $O/attn_dec_p78.raw.csv 2>/dev/null
rm -f $O/attn_dec_p78.ncu-rep
ls -la $O
