O=gpurun_out/r02; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q > $O/b_tests.log 2>&1
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 2 > $O/b_trace_dec2.jsonl 2>&1
BULLET_PDL=0 timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 2 > $O/b_trace_dec2_nopdl.jsonl 2>&1
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode pre --p 76 --k 1 > $O/b_trace_pre2.jsonl 2>&1
for pdl in 1 0; do
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 4 --time 20 --config sharegpt-8b > $O/b_pdl${pdl}_dec2.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode dec --p 84 --k 2 --reps 4 --time 10 --config arxiv-8b > $O/b_pdl${pdl}_dec3.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode pre --p 76 --k 1 --reps 4 --time 10 --config sharegpt-8b > $O/b_pdl${pdl}_pre2.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode corun --p 76 --k 8 --reps 4 --time 10 --config sharegpt-8b > $O/b_pdl${pdl}_co2.log 2>&1
done
BULLET_GEMM_KCHUNK=0 timeout 900 python scripts/precision_layer.py qwen2.5-14b llama3.1-70b --pre 1024,512 --dec 2000,17 --sample 192 > $O/b_prec_nokc_pre.jsonl 2>&1
echo done
