O=gpurun_out/r02; mkdir -p $O
for pf in 0 2 4 8; do
  BULLET_DEC_PF=$pf timeout 300 python scripts/attn_dec_bench.py --config arxiv-8b --kind 3 --sms 64 76 148 --tag pf$pf >> $O/r_attn_pf.jsonl 2>>$O/r_attn_pf.err
  BULLET_DEC_PF=$pf timeout 300 python scripts/attn_dec_bench.py --config sharegpt-8b --kind 3 --sms 64 72 148 --tag pf$pf >> $O/r_attn_pf.jsonl 2>>$O/r_attn_pf.err
done
for pf in 0 4 8 16; do
  BULLET_GEMM_PF=$pf timeout 300 python scripts/prof_step.py --mode dec --p 84 --k 4 --reps 4 --time 20 --config sharegpt-8b > $O/r_gemm_pf${pf}_dec2.log 2>&1
done
echo done
