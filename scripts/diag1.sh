cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for p in 80 0; do
  BULLET_GEMM_DEBUG=1 python scripts/prof_step.py --mode dec --p $p --k 4 --reps 3 --time 10 > gpurun_out/diag_dec_p$p.txt 2>&1
done
python scripts/prof_step.py --mode pre --p 80 --reps 3 --time 5 > gpurun_out/diag_pre_p80.txt 2>&1
python scripts/prof_step.py --mode pre --p 148 --reps 3 --time 5 > gpurun_out/diag_pre_p148.txt 2>&1
python scripts/prof_step.py --mode corun --p 80 --k 7 --reps 3 --time 10 > gpurun_out/diag_corun_p80.txt 2>&1
