O=gpurun_out/r02; mkdir -p $O
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/j_trace_dec2.jsonl 2>&1
for pdl in 1 0; do
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 4 --time 20 --config sharegpt-8b > $O/j_pdl${pdl}_dec2.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode dec --p 84 --k 2 --reps 4 --time 10 --config arxiv-8b > $O/j_pdl${pdl}_dec3.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode pre --p 76 --k 1 --reps 4 --time 10 --config sharegpt-8b > $O/j_pdl${pdl}_pre2.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode corun --p 76 --k 8 --reps 4 --time 10 --config sharegpt-8b > $O/j_pdl${pdl}_co2.log 2>&1
  BULLET_PDL=$pdl timeout 300 python scripts/prof_step.py --mode timesliced --p 148 --k 8 --reps 4 --time 10 --config sharegpt-8b > $O/j_pdl${pdl}_ts2.log 2>&1
done
timeout 900 python -m pytest tests -m gpu -x -q > $O/j_tests.log 2>&1
echo done
