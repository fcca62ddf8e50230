#!/bin/bash
# Q tiles by TMA in the prefill attention (tests + A/B vs the K/V-only build's numbers), decode GEMM traces
# with the accumulator-ready slot.
set -u
O=gpurun_out/s4; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_layer.py tests/test_gpu_kernels.py -k "attention or tma_kv or gqa_pair or mixed or chunk" -q -x > $O/tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/tests.log
for t in 1 0; do
  for cfg in arxiv-8b sharegpt-8b; do
    BULLET_PF5_TMA=$t timeout 300 python scripts/attn_pre_bench.py --config $cfg --sms 78 86 148 --reps 20 --tag "qkv-tma=$t" >> $O/attn_pre.jsonl 2>> $O/attn_pre.err
  done
done
cat $O/attn_pre.jsonl
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 2 > $O/trace_c2_p80.jsonl 2> $O/trace.err
timeout 300 python scripts/trace_step.py --config arxiv-8b --mode dec --p 78 --k 2 > $O/trace_c3_p78.jsonl 2>> $O/trace.err
echo done
