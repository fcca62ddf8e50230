#!/bin/bash
# Decode attention warps x stages with the TMA stream: 12 x 2 (default) vs 8 x 3 vs 16 x 1 (variant libs).
set -u
O=gpurun_out/${OUT:-s28}; mkdir -p $O
L=$PWD/paper_conf_asplos_0001xc0l026_b200
for rep in 1 2; do
  for v in default w8d3 w16d1; do
    for cfg in sharegpt-8b arxiv-8b; do
      if [ $v = default ]; then env -u BULLET_LIB timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "$v rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
      else BULLET_LIB=$L/libbullet_$v.so timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "$v rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err; fi
    done
  done
done
tail -3 $O/attn_dec.err
