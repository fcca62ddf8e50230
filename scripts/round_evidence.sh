#!/bin/bash
# One gpurun call: bench lines of configs 2 and 3, then the ncu captures at the
# splits the bench chose (scripts/capture_r01c.sh).  Writes gpurun_out/.
set -u
mkdir -p gpurun_out
timeout 900 python bench.py --config sharegpt-8b > gpurun_out/bench_sharegpt.json 2> gpurun_out/bench_sharegpt.err
timeout 1200 python bench.py --config arxiv-8b > gpurun_out/bench_arxiv.json 2> gpurun_out/bench_arxiv.err
split() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(d['config']['prefill_sm_count'], d['config']['decode_layer_steps'])" $1; }
read P2 K2 < <(split gpurun_out/bench_sharegpt.json)
read P3 K3 < <(split gpurun_out/bench_arxiv.json)
echo "splits: $P2 $K2 / $P3 $K3"
bash scripts/capture_r01c.sh $P2 $K2 $P3 $K3
