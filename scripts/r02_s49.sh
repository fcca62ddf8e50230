#!/bin/bash
# KC after the countdown fix: where the remaining cost is (merge skipped / stores skipped / one chunk).
set -u
O=gpurun_out/${OUT:-s49}; mkdir -p $O
run() { local tag=$1; shift; echo "== $tag" >> $O/prof.log; env "$@" timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 148 --config arxiv-8b >> $O/prof.log 2>&1; }
for rep in 1 2; do
  run bn128 BULLET_GEMM_PLAN_K2P=1,128,0 BULLET_GEMM_PLAN_K5P=1,128,0
  run kc256 BULLET_GEMM_KCHUNK=256
  run kc256_nomerge BULLET_GEMM_KCHUNK=256 BULLET_GEMM_EPI_DBG=16
  run kc512 BULLET_GEMM_KCHUNK=512
  run kc_one BULLET_GEMM_KCHUNK=256 BULLET_GEMM_EPI_DBG=32
done
grep -E "==|qkv" $O/prof.log
