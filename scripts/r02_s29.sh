#!/bin/bash
# Run-to-run spread of the bench lines on one box (3 x config 3, 2 x config 2).
set -u
O=gpurun_out/s29; mkdir -p $O
for i in 1 2 3; do timeout 900 python bench.py --no-cpu-baseline > $O/bench_arxiv_$i.json 2> $O/bench_arxiv_$i.err; echo "c3 $i rc=$?"; done
for i in 1 2; do timeout 900 python bench.py --config sharegpt-8b --no-cpu-baseline > $O/bench_sharegpt_$i.json 2> $O/bench_sharegpt_$i.err; echo "c2 $i rc=$?"; done
