set -u
O=gpurun_out/r02; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/base_smi.txt 2>&1
timeout 300 python scripts/prof_step.py --mode dec --p 80 --k 1 --reps 4 --config sharegpt-8b > $O/base_dec_c2_p80.log 2>&1
timeout 300 python scripts/prof_step.py --mode dec --p 84 --k 1 --reps 4 --config arxiv-8b > $O/base_dec_c3_p84.log 2>&1
timeout 600 python bench.py --config arxiv-8b --sweep --no-cpu-baseline > $O/base_bench3.json 2> $O/base_bench3.err
timeout 600 python bench.py --config sharegpt-8b --sweep --no-cpu-baseline > $O/base_bench2.json 2> $O/base_bench2.err
echo done
