#!/bin/bash
# Decode gate_up with 448-row tiles (two N = 224 MMAs, one wave on 64 SMs): parity, plan sweep, traces, bench.
set -u
O=gpurun_out/${OUT:-s26}; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" > $O/tests_k.log 2>&1; echo "gemm tests rc=$?"; tail -3 $O/tests_k.log
timeout 600 python -m pytest tests/test_gpu_layer.py -q -x -k "config2 or config3 or corun or knobs" > $O/tests_l.log 2>&1; echo "layer tests rc=$?"; tail -3 $O/tests_l.log
timeout 900 python scripts/decode_gemm_plans.py --config sharegpt-8b --p 84 80 --k 4 > $O/plans2.log 2>&1
timeout 900 python scripts/decode_gemm_plans.py --config arxiv-8b --p 78 --k 2 > $O/plans3.log 2>&1
grep gate_up $O/plans2.log $O/plans3.log
BULLET_GEMM_DEBUG=1 timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 2 > $O/trace_c2_p80.jsonl 2> $O/trace.err; grep "N=28672" $O/trace.err | sort | uniq -c
timeout 900 python bench.py --config sharegpt-8b > $O/bench_sharegpt.json 2> $O/bench_sharegpt.err; echo "bench2 rc=$?"
echo done
