O=gpurun_out/r02; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_tp_peer.py tests/test_gpu_layer.py::test_fused_qkv_pool_vs_oracle "tests/test_gpu_kernels.py::test_attention_vs_oracle" -x -q > $O/a_tests.log 2>&1
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 2 > $O/a_trace_dec2.jsonl 2>&1
timeout 300 python scripts/trace_step.py --config arxiv-8b --mode dec --p 84 --k 1 > $O/a_trace_dec3.jsonl 2>&1
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode pre --p 76 --k 1 > $O/a_trace_pre2.jsonl 2>&1
for kc in 0 256; do
  BULLET_GEMM_KCHUNK=$kc timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 1 --reps 4 --time 20 --config sharegpt-8b > $O/a_kc${kc}_dec2.log 2>&1
  BULLET_GEMM_KCHUNK=$kc timeout 300 python scripts/prof_step.py --mode pre --p 76 --k 1 --reps 4 --time 10 --config sharegpt-8b > $O/a_kc${kc}_pre2.log 2>&1
  BULLET_GEMM_KCHUNK=$kc timeout 300 python scripts/prof_step.py --mode pre --p 84 --k 1 --reps 3 --time 5 --config arxiv-8b > $O/a_kc${kc}_pre3.log 2>&1
done
echo done
