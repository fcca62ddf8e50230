#!/bin/bash
# Prefill GEMM epilogue cost (config 3, 78 SMs): per-kernel times with diagnostic switches
# (BULLET_GEMM_EPI_DBG: 1 no SiLU math, 2 no stores, 4 no residual loads, 8 no RoPE loads; wrong results).
set -u
O=gpurun_out/s24; mkdir -p $O
for rep in 1 2; do
for d in 0 2 4 6 8 15; do
  echo "== dbg=$d rep=$rep" >> $O/prof.log
  BULLET_GEMM_EPI_DBG=$d timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 78 --config arxiv-8b >> $O/prof.log 2>&1
done
done
cat $O/prof.log | grep -E "==|qkv|o_proj|gate_up|down|step"
