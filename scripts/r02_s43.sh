#!/bin/bash
# Split decision with the 6 % tie window (R-23) and the damped, bounded feedback: repeated bench lines.
set -u
O=gpurun_out/s43; mkdir -p $O
for i in 1 2 3 4; do timeout 900 python bench.py --no-cpu-baseline > $O/bench_arxiv_$i.json 2> $O/bench_arxiv_$i.err; echo "c3 $i rc=$?"; done
for i in 1 2; do timeout 900 python bench.py --config sharegpt-8b --no-cpu-baseline > $O/bench_sharegpt_$i.json 2> $O/bench_sharegpt_$i.err; echo "c2 $i rc=$?"; done
