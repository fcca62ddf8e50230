#!/bin/bash
set -u
O=gpurun_out/s42; mkdir -p $O
run() { local tag=$1; shift; echo "== $tag" >> $O/prof.log; env "$@" timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 148 --config arxiv-8b >> $O/prof.log 2>&1; }
for rep in 1 2; do
  run bn128 BULLET_GEMM_PLAN_K2P=1,128,0 BULLET_GEMM_PLAN_K5P=1,128,0
  run kc_one BULLET_GEMM_KCHUNK=256 BULLET_GEMM_EPI_DBG=32
  run kc_one_2st BULLET_GEMM_KCHUNK=256 BULLET_GEMM_EPI_DBG=96
  run kc256_2st BULLET_GEMM_KCHUNK=256 BULLET_GEMM_EPI_DBG=64
done
grep -E "==|qkv|o_proj" $O/prof.log
