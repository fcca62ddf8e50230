O=gpurun_out/r02; mkdir -p $O
BULLET_GEMM_DEBUG=1 timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/d_trace_dec2.jsonl 2>$O/d_trace_dec2.err
for plan in "1,256,0" "1,128,0" "1,128,1"; do
  BULLET_GEMM_PLAN=$plan timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/d_trace_dec2_$plan.jsonl 2>&1
done
timeout 900 python -m pytest tests -m gpu -x -q > $O/d_tests.log 2>&1
echo done
