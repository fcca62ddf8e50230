#!/bin/bash
# Full GPU suite + smoke + bench lines of configs 3 (default) and 2 on the current kernels.
set -u
O=gpurun_out/${OUT:-s10}; mkdir -p $O
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
timeout 900 python bench.py > $O/bench_arxiv.json 2> $O/bench_arxiv.err; echo "bench3 rc=$?"
timeout 900 python bench.py --config sharegpt-8b > $O/bench_sharegpt.json 2> $O/bench_sharegpt.err; echo "bench2 rc=$?"
echo done
