O=gpurun_out/r02; mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_layer.py -k "pool" -x -q > $O/e_pool.log 2>&1
BULLET_GEMM_DEBUG=1 timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/e_trace_dec2.jsonl 2>$O/e_trace_dec2.err
BULLET_GEMM_DEBUG=1 timeout 300 python scripts/trace_step.py --config arxiv-8b --mode dec --p 84 --k 1 > $O/e_trace_dec3.jsonl 2>$O/e_trace_dec3.err
timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 4 --time 20 --config sharegpt-8b > $O/e_dec2.log 2>&1
timeout 300 python scripts/prof_step.py --mode pre --p 76 --k 1 --reps 4 --time 10 --config sharegpt-8b > $O/e_pre2.log 2>&1
echo done
