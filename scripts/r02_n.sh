O=gpurun_out/r02; mkdir -p $O
for mb in 32 64 128; do
  BULLET_GEMM_BAND_MB=$mb timeout 300 python scripts/prof_step.py --mode corun --p 76 --k 8 --reps 4 --time 20 --config sharegpt-8b > $O/n_band${mb}_co2.log 2>&1
  BULLET_GEMM_BAND_MB=$mb timeout 300 python scripts/prof_step.py --mode corun --p 84 --k 5 --reps 4 --time 10 --config arxiv-8b > $O/n_band${mb}_co3.log 2>&1
done
timeout 900 python bench.py --sweep --no-cpu-baseline > $O/n_bench3.json 2> $O/n_bench3.err
timeout 900 python bench.py --config sharegpt-8b --sweep --no-cpu-baseline > $O/n_bench2.json 2> $O/n_bench2.err
timeout 900 python -m pytest tests -m gpu -q > $O/n_tests.log 2>&1
echo done
