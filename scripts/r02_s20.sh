#!/bin/bash
# Prefill down GEMM (K = 14336) L2 working set: plan / band variants, co-run step time at config 3's split
# (interleaved repeats) and the down launch alone.
set -u
O=gpurun_out/s20; mkdir -p $O
run() {  # tag, env...
  local tag=$1; shift
  env "$@" timeout 300 python scripts/prof_step.py --mode corun --p 78 --k 5 --config arxiv-8b --reps 1 --quiet --time 10 > $O/corun_$tag.log 2>&1
  echo "{\"tag\": \"$tag\", \"corun\": \"$(grep -h 'timed' $O/corun_$tag.log | tail -1)\"}" >> $O/res.jsonl
}
for rep in 1 2 3; do
  run base
  run bn128_b32 BULLET_GEMM_PLAN_K8P=1,128,1 BULLET_GEMM_BAND_MB_K8=32
  run b32 BULLET_GEMM_BAND_MB_K8=32
  run b128 BULLET_GEMM_BAND_MB_K8=128
done
cat $O/res.jsonl
F="ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none"
for v in "base" "bn128_b32 BULLET_GEMM_PLAN_K8P=1,128,1 BULLET_GEMM_BAND_MB_K8=32" "b32 BULLET_GEMM_BAND_MB_K8=32" "b128 BULLET_GEMM_BAND_MB_K8=128"; do
  set -- $v; tag=$1; shift
  env "$@" timeout 300 $F -k regex:k_gemm_tc -s 7 -c 1 --csv python scripts/prof_step.py --reps 2 --quiet --mode pre --p 78 --config arxiv-8b > $O/ncu_down_$tag.csv 2>&1
done
tail -n 6 $O/ncu_down_*.csv
