#!/bin/bash
# Decode attention: K / V blocks by TMA boxes (BULLET_DEC_TMA=1) vs cp.async, interleaved;
# no-math stream ceiling (BULLET_DBG=1); parity tests; decode traces.
set -u
O=gpurun_out/${OUT:-s11}; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_layer.py -q -x -k "decode or attention or long or layer" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
for rep in 1 2; do
for sp in 1 0; do
  for cfg in sharegpt-8b arxiv-8b; do
    BULLET_DEC_TMA=$sp timeout 300 python scripts/attn_dec_bench.py --config $cfg --kind 3 --sms 64 70 148 --reps 10 --tag "tma=$sp rep=$rep" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
  done
done
done
for sp in 1 0; do
  BULLET_DBG=1 BULLET_DEC_TMA=$sp timeout 300 python scripts/attn_dec_bench.py --config arxiv-8b --kind 3 --sms 64 70 --reps 10 --tag "nomath tma=$sp" >> $O/attn_dec.jsonl 2>> $O/attn_dec.err
done
cat $O/attn_dec.jsonl
echo done
