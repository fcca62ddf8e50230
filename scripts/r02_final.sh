#!/bin/bash
# Round-2 closing evidence: bench lines (configs 3 and 2), ncu captures at their splits, launch lists,
# full GPU suite + smoke.  Writes gpurun_out/final/ and gpurun_out/ncu3/.
set -u
O=gpurun_out/final; mkdir -p $O
timeout 900 python bench.py > $O/bench_arxiv.json 2> $O/bench_arxiv.err; echo "bench3 rc=$?"
timeout 900 python bench.py --config sharegpt-8b > $O/bench_sharegpt.json 2> $O/bench_sharegpt.err; echo "bench2 rc=$?"
split() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(d['config']['prefill_sm_count'], d['config']['decode_layer_steps'])" $1; }
read P3 K3 < <(split $O/bench_arxiv.json)
read P2 K2 < <(split $O/bench_sharegpt.json)
echo "splits: $P2 $K2 / $P3 $K3"
KEEP_REP="" bash scripts/capture_r02b.sh $P2 $K2 $P3 $K3 > $O/capture.log 2>&1; echo "capture rc=$?"
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
echo done
