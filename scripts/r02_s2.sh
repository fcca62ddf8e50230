#!/bin/bash
# Prefill attention: TMA-fed K/V tiles vs cp.async gathers (A/B, interleaved), parity tests, bench.
set -u
O=gpurun_out/s2; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_layer.py -k "tma_kv or gqa_pair" tests/test_gpu_kernels.py -k "attention or tma_kv or gqa_pair" -q -x > $O/tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/tests.log
for rep in 1 2; do
for t in 1 0; do
  for cfg in arxiv-8b sharegpt-8b; do
    BULLET_PF5_TMA=$t timeout 300 python scripts/attn_pre_bench.py --config $cfg --sms 78 86 148 --reps 20 --tag "tma=$t rep=$rep" >> $O/attn_pre.jsonl 2>> $O/attn_pre.err
  done
done
done
cat $O/attn_pre.jsonl
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
tail -c 300 $O/bench.json
