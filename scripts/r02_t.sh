O=gpurun_out/r02; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q > $O/t_tests.log 2>&1
timeout 900 python scripts/decode_gemm_plans.py --config sharegpt-8b --p 80 84 --k 4 > $O/t_plans2.log 2>&1
timeout 900 python scripts/decode_gemm_plans.py --config arxiv-8b --p 84 --k 2 > $O/t_plans3.log 2>&1
echo done
