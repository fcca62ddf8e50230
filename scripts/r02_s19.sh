#!/bin/bash
# ncu of the prefill QKV / O-proj / down GEMMs (config 3, 78 SMs): why below gate_up's rate.
set -u
O=gpurun_out/s19; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
# prefill layer GEMM order: qkv(0) o_proj(1) gate_up(2) down(3); prof_step runs warm-up reps first
i=0
for g in qkv oproj gateup down; do
  timeout 300 $F -k regex:k_gemm_tc -s $((4 + i)) -c 1 -o $O/c3_${g}_pre_p78 python scripts/prof_step.py --reps 2 --quiet --mode pre --p 78 --config arxiv-8b > $O/$g.log 2>&1
  ncu -i $O/c3_${g}_pre_p78.ncu-rep --page raw --csv > $O/c3_${g}_pre_p78.raw.csv 2>/dev/null
  ncu -i $O/c3_${g}_pre_p78.ncu-rep --page source --csv --print-source sass > $O/c3_${g}_pre_p78.sass.csv 2>/dev/null
  rm -f $O/c3_${g}_pre_p78.ncu-rep
  i=$((i + 1))
done
ls -la $O
