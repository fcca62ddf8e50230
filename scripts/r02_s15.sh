#!/bin/bash
# tcgen05 decode attention: where the time goes (BULLET_DBG diagnostic bits, wrong results).
set -u
O=gpurun_out/${OUT:-s15}; mkdir -p $O
for d in 0 4 8 12 16 32; do
  BULLET_DBG=$d timeout 300 python scripts/attn_dec_bench.py --config arxiv-8b --kind 3 --sms 70 148 --reps 10 --tag "dbg=$d" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
done
cat $O/attn_dec.jsonl; tail -3 $O/attn_dec.err
