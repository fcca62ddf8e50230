#!/bin/bash
# Round-2 final ncu evidence (r02b: TMA-fed attentions, decode GEMM epilogues): all four decode GEMMs and the decode attention at the
# bench splits of configs 2 and 3, the prefill gate_up (the bench's dominant
# tensor kernel) and prefill attention, and the launch lists of the bench
# commands.  Run under gpurun (one GPU).  Writes gpurun_out/ncu2/.
#   bash scripts/capture_r02.sh P2 K2 P3 K3
set -u
P2=${1:-76}; K2=${2:-8}; P3=${3:-84}; K3=${4:-5}
O=gpurun_out/ncu3; mkdir -p $O
F="ncu --set full --clock-control none --import-source on"
cap() { # name, kernel regex, skip, prof_step args...  (raw metrics exported as csv; the .ncu-rep is
         # dropped unless KEEP_REP names it: gpurun brings back <= 64 MiB)
  local name=$1 k=$2 s=$3; shift 3
  timeout 300 $F -k regex:$k -s $s -c 1 -o $O/$name python scripts/prof_step.py --reps 2 --quiet "$@" > $O/$name.log 2>&1
  ncu -i $O/$name.ncu-rep --page raw --csv > $O/$name.raw.csv 2>/dev/null
  case " ${KEEP_REP:-} " in *" $name "*) ;; *) rm -f $O/$name.ncu-rep ;; esac
}
# decode layer GEMM order: qkv(0) o_proj(1) gate_up(2) down(3) (second step: +4)
i=0
for g in qkv oproj gateup down; do
  cap r02b_c2_${g}_dec_p$P2 k_gemm_tc $((4 + i)) --mode dec --p $P2 --config sharegpt-8b
  cap r02b_c3_${g}_dec_p$P3 k_gemm_tc $((4 + i)) --mode dec --p $P3 --config arxiv-8b
  i=$((i + 1))
done
cap r02b_c2_attn_dec_p$P2   k_attn_decode   1 --mode dec --p $P2 --config sharegpt-8b
cap r02b_c3_attn_dec_p$P3   k_attn_decode   1 --mode dec --p $P3 --config arxiv-8b
cap r02b_c2_gateup_pre_p$P2 k_gemm_tc       6 --mode pre --p $P2 --config sharegpt-8b
cap r02b_c3_gateup_pre_p$P3 k_gemm_tc       6 --mode pre --p $P3 --config arxiv-8b
cap r02b_c3_attn_pre_p148   k_attn_prefill5 1 --mode pre --p 148 --config arxiv-8b
cap r02b_c3_attn_pre_p$P3   k_attn_prefill5 1 --mode pre --p $P3 --config arxiv-8b
cap r02b_c2_attn_pre_p$P2   k_attn_prefill5 1 --mode pre --p $P2 --config sharegpt-8b
for spec in "sharegpt-8b $P2 $K2" "arxiv-8b $P3 $K3"; do
  set -- $spec
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 4000 --csv \
    --log-file $O/r02b_launches_$1.csv python bench.py --config $1 --p $2 --k $3 --steps 2 --warmup 3 \
    --no-cpu-baseline --no-sweep --feedback 0 > $O/r02b_launches_$1.log 2>&1
done
ls -la $O
