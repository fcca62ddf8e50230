#!/bin/bash
# KC GEMM with four TMEM accumulator stages: cost vs plain tiles, parity (KC paths), simulated-TP prefill.
set -u
O=gpurun_out/${OUT:-s32}; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_tp_peer.py -q -x -k "accumulation or gemm or peer" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/tests.log
run() { local tag=$1; shift; echo "== $tag" >> $O/prof.log; env "$@" timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 148 --config arxiv-8b >> $O/prof.log 2>&1; }
for rep in 1 2; do
  run default
  run bn128 BULLET_GEMM_PLAN_K2P=1,128,0 BULLET_GEMM_PLAN_K5P=1,128,0
  run kc256 BULLET_GEMM_KCHUNK=256
done
grep -E "==|qkv|o_proj" $O/prof.log
CUDA_DEVICE_MAX_CONNECTIONS=32 timeout 600 python scripts/tp_sim_bench.py --config qwen14b-tp2 --reps 10 > $O/tp_sim.jsonl 2> $O/tp_sim.err; cat $O/tp_sim.jsonl | cut -c1-200
