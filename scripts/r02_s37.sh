#!/bin/bash
# ncu source view of the prefill QKV GEMM: KC (256-K chunks) vs plain 128-wide tiles (config 3, 148 SMs).
set -u
O=gpurun_out/s37; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
for v in "kc BULLET_GEMM_KCHUNK=256" "bn128 BULLET_GEMM_PLAN_K2P=1,128,0"; do
  set -- $v; tag=$1; shift
  env "$@" timeout 300 $F -k regex:k_gemm_tc -s 4 -c 1 -o $O/qkv_$tag python scripts/prof_step.py --reps 2 --quiet --mode pre --p 148 --config arxiv-8b > $O/$tag.log 2>&1
  ncu -i $O/qkv_$tag.ncu-rep --page raw --csv > $O/qkv_$tag.raw.csv 2>/dev/null
  ncu -i $O/qkv_$tag.ncu-rep --page source --csv --print-source sass > $O/qkv_$tag.sass.csv 2>/dev/null
  rm -f $O/qkv_$tag.ncu-rep
done
ls -la $O
