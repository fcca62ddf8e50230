#!/bin/bash
# Round-1 ncu evidence (run under gpurun, one GPU). Writes gpurun_out/ncu/.
set -u
O=gpurun_out/ncu; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
cap() { # name, kernel regex, skip, prof_step args...
  local name=$1 k=$2 s=$3; shift 3
  timeout 300 $F -k regex:$k -s $s -c 1 -o $O/$name python scripts/prof_step.py --reps 2 --quiet "$@" > $O/$name.log 2>&1
}
cap r01_c2_gateup_pre_p80   k_gemm_tc        2 --mode pre --p 80 --config sharegpt-8b
cap r01_c2_attn_pre_p148    k_attn_prefill5  0 --mode pre --p 148 --config sharegpt-8b
cap r01_c2_attn_dec_p80     k_attn_decode    0 --mode dec --p 80 --config sharegpt-8b
cap r01_c2_gateup_dec_p80   k_gemm_tc        2 --mode dec --p 80 --config sharegpt-8b
cap r01_c3_attn_dec_p88     k_attn_decode    0 --mode dec --p 88 --config arxiv-8b
cap r01_c3_attn_pre_p148    k_attn_prefill5  0 --mode pre --p 148 --config arxiv-8b
cap r01_c3_gateup_pre_p88   k_gemm_tc        2 --mode pre --p 88 --config arxiv-8b
# launch lists of the bench commands (the judged configuration, split fixed)
for spec in "sharegpt-8b 80 7" "arxiv-8b 88 4"; do
  set -- $spec
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 2000 --csv \
    --log-file $O/r01_launches_$1.csv python bench.py --config $1 --p $2 --k $3 --steps 2 --warmup 3 \
    --no-cpu-baseline > $O/r01_launches_$1.log 2>&1
done
ls -la $O
