#!/bin/bash
# Prefill attention MMA issuers: per-tile descriptors + offsets vs per-MMA descriptor builds (A/B, variant lib).
set -u
O=gpurun_out/s48; mkdir -p $O
V=$PWD/paper_conf_asplos_0001xc0l026_b200/libbullet_olddesc.so
for rep in 1 2; do
  for v in new old; do
    for cfg in arxiv-8b sharegpt-8b; do
      if [ $v = old ]; then BULLET_LIB=$V timeout 300 python scripts/attn_pre_bench.py --config $cfg --sms 78 148 --reps 20 --tag "$v" >> $O/attn_pre.jsonl 2>> $O/attn_pre.err
      else timeout 300 python scripts/attn_pre_bench.py --config $cfg --sms 78 148 --reps 20 --tag "$v" >> $O/attn_pre.jsonl 2>> $O/attn_pre.err; fi
    done
  done
done
timeout 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_layer.py -q -x -k "attention or tma_kv or gqa_pair" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
