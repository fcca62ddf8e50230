#!/bin/bash
# Prefill attention with 128-key tiles (BULLET_PF5_BKV=128: one S buffer per query tile): parity, A/B.
set -u
O=gpurun_out/${OUT:-s22}; mkdir -p $O
BULLET_PF5_BKV=128 timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention_vs_oracle" > $O/tests_k.log 2>&1; echo "kernel tests rc=$?"; tail -12 $O/tests_k.log
BULLET_PF5_BKV=128 timeout 900 python -m pytest tests/test_gpu_layer.py -q -x > $O/tests_l.log 2>&1; echo "layer tests rc=$?"; tail -3 $O/tests_l.log
for rep in 1 2; do
  for bkv in 128 64; do
    for cfg in arxiv-8b sharegpt-8b; do
      BULLET_PF5_BKV=$bkv timeout 300 python scripts/attn_pre_bench.py --config $cfg --sms 78 86 148 --reps 20 --tag "bkv=$bkv rep=$rep" >> $O/attn_pre.jsonl 2>> $O/attn_pre.err
    done
  done
done
cat $O/attn_pre.jsonl; tail -3 $O/attn_pre.err
