cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/d2_smoke.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/d2_pytest.log 2>&1
python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 3 --time 10 > gpurun_out/d2_dec_p80.txt 2>&1
python scripts/prof_step.py --mode pre --p 148 --reps 3 --time 5 > gpurun_out/d2_pre_p148.txt 2>&1
timeout 600 python scripts/decode_gemm_plans.py --p 80 0 > gpurun_out/d2_plans.txt 2>&1
