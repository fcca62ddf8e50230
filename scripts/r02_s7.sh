#!/bin/bash
# Residual loads batched before the stores (resid aliases out): traces A/B coalesced vs per-row epilogue.
set -u
O=gpurun_out/${OUT:-s7}; mkdir -p $O
for rep in 1 2; do
for c in 1 0; do
  for cfg in "sharegpt-8b 80" "arxiv-8b 78"; do
    set -- $cfg
    echo "{\"variant\": \"coal=$c rep=$rep\"}" >> $O/trace_$1.jsonl
    BULLET_GEMM_EPI_COAL=$c timeout 300 python scripts/trace_step.py --config $1 --mode dec --p $2 --k 2 >> $O/trace_$1.jsonl 2>> $O/trace.err
  done
done
done
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
echo done
