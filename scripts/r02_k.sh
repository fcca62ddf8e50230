O=gpurun_out/r02; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q > $O/k_tests.log 2>&1
BULLET_GEMM_DEBUG=1 timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/k_trace_dec2.jsonl 2>$O/k_trace_dec2.err
timeout 900 python bench.py --sweep --no-cpu-baseline > $O/k_bench3.json 2> $O/k_bench3.err
timeout 900 python bench.py --config sharegpt-8b --sweep --no-cpu-baseline > $O/k_bench2.json 2> $O/k_bench2.err
echo done
