#!/bin/bash
# Round-1 closing capture (after the two-level-accumulation template was added
# to k_gemm_tc): the bench's dominant kernel (prefill gate_up at the bench
# split), the decode attention, and the launch list of the config-2 bench
# command.  Run under gpurun (one GPU).  Writes gpurun_out/ncu/.
set -u
P2=${1:-76}; K2=${2:-8}
O=gpurun_out/ncu; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
cap() { local name=$1 k=$2 s=$3; shift 3
  timeout 300 $F -k regex:$k -s $s -c 1 -o $O/$name python scripts/prof_step.py --reps 2 --quiet "$@" > $O/$name.log 2>&1; }
cap r01d_c2_gateup_pre_p$P2 k_gemm_tc     2 --mode pre --p $P2 --config sharegpt-8b
cap r01d_c2_attn_dec_p$P2   k_attn_decode 0 --mode dec --p $P2 --config sharegpt-8b
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 4000 --csv \
  --log-file $O/r01d_launches_sharegpt-8b.csv python bench.py --config sharegpt-8b --p $P2 --k $K2 --steps 2 --warmup 3 \
  --no-cpu-baseline > $O/r01d_launches_sharegpt-8b.log 2>&1
ls -la $O
