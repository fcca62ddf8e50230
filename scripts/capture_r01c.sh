#!/bin/bash
# Round-1 (third pass) ncu evidence after the fused all-reduce, kernel preload, fused RMSNorm tail and
# attention consumer groups.  Run under gpurun (one GPU).  Writes gpurun_out/ncu/.
#   bash scripts/capture_r01c.sh P2 K2 P3 K3     (bench splits of config 2 / config 3)
set -u
P2=${1:-80}; K2=${2:-8}; P3=${3:-80}; K3=${4:-5}
O=gpurun_out/ncu; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
cap() { # name, kernel regex, skip, prof_step args...
  local name=$1 k=$2 s=$3; shift 3
  timeout 300 $F -k regex:$k -s $s -c 1 -o $O/$name python scripts/prof_step.py --reps 2 --quiet "$@" > $O/$name.log 2>&1
}
# decode layer GEMM order: qkv(0) o_proj(1) gate_up(2) down(3); prefill the same
cap r01c_c2_gateup_pre_p$P2   k_gemm_tc        2 --mode pre --p $P2 --config sharegpt-8b
cap r01c_c2_qkv_pre_p148      k_gemm_tc        0 --mode pre --p 148 --config sharegpt-8b
cap r01c_c2_attn_pre_p148     k_attn_prefill5  0 --mode pre --p 148 --config sharegpt-8b
cap r01c_c2_attn_dec_p$P2     k_attn_decode    0 --mode dec --p $P2 --config sharegpt-8b
cap r01c_c2_gateup_dec_p$P2   k_gemm_tc        2 --mode dec --p $P2 --config sharegpt-8b
cap r01c_c2_qkv_dec_p$P2      k_gemm_tc        0 --mode dec --p $P2 --config sharegpt-8b
cap r01c_c3_attn_dec_p$P3     k_attn_decode    0 --mode dec --p $P3 --config arxiv-8b
cap r01c_c3_attn_pre_p148     k_attn_prefill5  0 --mode pre --p 148 --config arxiv-8b
cap r01c_c3_gateup_pre_p$P3   k_gemm_tc        2 --mode pre --p $P3 --config arxiv-8b
# launch lists of the bench commands at the bench's splits
for spec in "sharegpt-8b $P2 $K2" "arxiv-8b $P3 $K3"; do
  set -- $spec
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 4000 --csv \
    --log-file $O/r01c_launches_$1.csv python bench.py --config $1 --p $2 --k $3 --steps 2 --warmup 3 \
    --no-cpu-baseline > $O/r01c_launches_$1.log 2>&1
done
ls -la $O
