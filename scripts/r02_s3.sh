#!/bin/bash
# Decode layer-step at config 2 on 68 / 64 SMs (verdict target <= 260 us on 68), per-CTA traces of the
# decode GEMMs, ncu of the TMA-fed prefill attention at 8k on 148 SMs.
set -u
O=gpurun_out/s3; mkdir -p $O
timeout 600 python scripts/decode_gemm_plans.py --config sharegpt-8b --p 80 84 --k 4 > $O/plans2.log 2>&1
for p in 80 84; do
  timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p $p --k 2 > $O/trace_c2_p$p.jsonl 2> $O/trace.err
done
timeout 300 python scripts/trace_step.py --config arxiv-8b --mode dec --p 78 --k 2 > $O/trace_c3_p78.jsonl 2>> $O/trace.err
F="ncu --set full --clock-control none --import-source on"
timeout 400 $F -k regex:k_attn_prefill5 -s 1 -c 1 -o $O/attn_pre_p148 python scripts/prof_step.py --reps 2 --quiet --mode pre --p 148 --config arxiv-8b > $O/attn_pre_ncu.log 2>&1
ncu -i $O/attn_pre_p148.ncu-rep --page raw --csv > $O/attn_pre_p148.raw.csv 2>/dev/null
ncu -i $O/attn_pre_p148.ncu-rep --page source --csv > $O/attn_pre_p148.source.csv 2>/dev/null
rm -f $O/attn_pre_p148.ncu-rep
echo done
