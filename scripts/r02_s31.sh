#!/bin/bash
# Two-level accumulation cost (R-4e): prefill QKV / O-proj with KC (kc 256, 512), vs plain bn=128 and the
# default bn=256, config 3 prefill on 148 SMs.
set -u
O=gpurun_out/s31; mkdir -p $O
run() { local tag=$1; shift; echo "== $tag" >> $O/prof.log; env "$@" timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 148 --config arxiv-8b >> $O/prof.log 2>&1; }
for rep in 1 2; do
  run default
  run bn128 BULLET_GEMM_PLAN_K2P=1,128,0 BULLET_GEMM_PLAN_K5P=1,128,0
  run kc256 BULLET_GEMM_KCHUNK=256
  run kc512 BULLET_GEMM_KCHUNK=512
  run kc1024 BULLET_GEMM_KCHUNK=1024
done
grep -E "==|qkv|o_proj" $O/prof.log
