#!/bin/bash
# tcgen05 decode attention (attn_decode5.cu): parity tests, A/B vs the mma.sync kernel (BULLET_DEC_KERNEL=3).
set -u
O=gpurun_out/${OUT:-s14}; mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "decode" > $O/tests_k.log 2>&1; echo "kernel tests rc=$?"; tail -15 $O/tests_k.log
timeout 600 python -m pytest tests/test_gpu_layer.py -q -x -k "decode or long or layer" > $O/tests_l.log 2>&1; echo "layer tests rc=$?"; tail -3 $O/tests_l.log
for rep in 1 2; do
for k in 5 3; do
  for cfg in sharegpt-8b arxiv-8b; do
    BULLET_DEC_KERNEL=$k timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "kernel=$k rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
  done
done
done
cat $O/attn_dec.jsonl; tail -5 $O/attn_dec.err
echo done
