#!/bin/bash
# MMA issuer: per-stage descriptors (+ address-field offsets) vs 8 descriptor builds per k-block; A/B with a
# variant lib of the previous build, interleaved.
set -u
O=gpurun_out/s47; mkdir -p $O
V=$PWD/paper_conf_asplos_0001xc0l026_b200/libbullet_olddesc.so
for rep in 1 2; do
  for v in new old; do
    if [ $v = old ]; then export BULLET_LIB=$V; else unset BULLET_LIB; fi
    echo "== $v rep=$rep" >> $O/prof.log
    timeout 300 python scripts/prof_step.py --reps 3 --mode pre --p 78 --config arxiv-8b >> $O/prof.log 2>&1
    timeout 300 python scripts/prof_step.py --reps 3 --mode dec --p 84 --k 4 --config sharegpt-8b >> $O/prof.log 2>&1
    timeout 300 python scripts/prof_step.py --reps 3 --mode dec --p 78 --k 2 --config arxiv-8b >> $O/prof.log 2>&1
  done
done
unset BULLET_LIB
timeout 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
