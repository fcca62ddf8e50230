cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/d4_smoke.log 2>&1
timeout 600 python -m pytest tests -m gpu -q > gpurun_out/d4_pytest.log 2>&1
for v in 5 3; do for nw in 16 12; do
BULLET_DEC_ATTN=$v BULLET_DEC2_WARPS=$nw python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 3 --time 10 > gpurun_out/d4_dec_p80_k${v}_w$nw.txt 2>&1
BULLET_DEC_ATTN=$v BULLET_DEC2_WARPS=$nw python scripts/prof_step.py --mode dec --p 0 --k 4 --reps 3 --time 10 > gpurun_out/d4_dec_p0_k${v}_w$nw.txt 2>&1
BULLET_DEC_ATTN=$v BULLET_DEC2_WARPS=$nw python scripts/prof_step.py --config arxiv-8b --mode dec --p 88 --k 2 --reps 3 --time 6 > gpurun_out/d4_c3dec_p88_k${v}_w$nw.txt 2>&1
done; done
