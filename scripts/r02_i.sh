O=gpurun_out/r02; mkdir -p $O
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/i_trace_dec2.jsonl 2>&1
timeout 300 python scripts/trace_step.py --config arxiv-8b --mode dec --p 84 --k 1 > $O/i_trace_dec3.jsonl 2>&1
timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 4 --reps 4 --time 20 --config sharegpt-8b > $O/i_dec2.log 2>&1
timeout 300 python scripts/prof_step.py --mode dec --p 84 --k 2 --reps 4 --time 10 --config arxiv-8b > $O/i_dec3.log 2>&1
timeout 300 python scripts/prof_step.py --mode pre --p 76 --k 1 --reps 4 --time 10 --config sharegpt-8b > $O/i_pre2.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/i_tests.log 2>&1
echo done
