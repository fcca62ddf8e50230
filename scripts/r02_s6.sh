#!/bin/bash
# Coalesced EPI_RESID / EPI_SILU epilogue + MUFU SiLU: parity tests, per-CTA traces A/B (BULLET_GEMM_EPI_COAL), bench.
set -u
O=gpurun_out/s6; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_layer.py -q -x > $O/tests.log 2>&1; echo "tests rc=$?"; tail -3 $O/tests.log
for rep in 1 2; do
for c in 1 0; do
  for cfg in "sharegpt-8b 80" "arxiv-8b 78"; do
    set -- $cfg
    echo "{\"variant\": \"coal=$c rep=$rep\"}" >> $O/trace_$1.jsonl
    BULLET_GEMM_EPI_COAL=$c timeout 300 python scripts/trace_step.py --config $1 --mode dec --p $2 --k 2 >> $O/trace_$1.jsonl 2>> $O/trace.err
  done
done
done
timeout 900 python bench.py --config sharegpt-8b > $O/bench_sharegpt.json 2> $O/bench_sharegpt.err; echo "bench2 rc=$?"
timeout 900 python bench.py > $O/bench_arxiv.json 2> $O/bench_arxiv.err; echo "bench3 rc=$?"
echo done
