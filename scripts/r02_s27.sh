#!/bin/bash
# Bench lines with the refit performance model (configs 3 and 2).
set -u
O=gpurun_out/s27; mkdir -p $O
timeout 900 python bench.py > $O/bench_arxiv.json 2> $O/bench_arxiv.err; echo "bench3 rc=$?"
timeout 900 python bench.py --config sharegpt-8b > $O/bench_sharegpt.json 2> $O/bench_sharegpt.err; echo "bench2 rc=$?"
