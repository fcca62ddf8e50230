#!/bin/bash
# Decode GEMM epilogue decomposition: L2 prefetch of the epilogue inputs on/off, and diagnostic builds
# without SiLU math (1), stores (2), residual loads (4), RoPE-table loads (8).
set -u
O=gpurun_out/s5; mkdir -p $O
for v in "PF=1 DBG=0" "PF=0 DBG=0" "PF=0 DBG=1" "PF=0 DBG=2" "PF=0 DBG=4" "PF=0 DBG=8" "PF=0 DBG=15"; do
  set -- $v; pf=${1#PF=}; dbg=${2#DBG=}
  for cfg in "sharegpt-8b 80" "arxiv-8b 78"; do
    set -- $cfg
    echo "{\"variant\": \"pf=$pf dbg=$dbg\"}" >> $O/trace_$1.jsonl
    BULLET_GEMM_EPI_PF=$pf BULLET_GEMM_EPI_DBG=$dbg timeout 300 python scripts/trace_step.py --config $1 --mode dec --p $2 --k 2 >> $O/trace_$1.jsonl 2>> $O/trace.err
  done
done
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_layer.py -q -x > $O/tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/tests.log
echo done
