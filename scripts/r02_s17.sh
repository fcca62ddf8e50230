#!/bin/bash
# Decode attention: four QK accumulation chains (variant lib) vs two, interleaved.
set -u
O=gpurun_out/${OUT:-s17}; mkdir -p $O
V=$PWD/paper_conf_asplos_0001xc0l026_b200/libbullet_qk4.so
for rep in 1 2; do
  for cfg in sharegpt-8b arxiv-8b; do
    BULLET_LIB=$V timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "qk4 rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
    timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "qk2 rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
  done
done
cat $O/attn_dec.jsonl; tail -3 $O/attn_dec.err
