#!/bin/bash
# Row-grid kernels without PDL: smid gating invariants repeated, full GPU suite, smoke, bench (config 3).
set -u
O=gpurun_out/s23; mkdir -p $O
for i in 1 2 3 4 5 6; do
  timeout 300 python -m pytest tests/test_gpu_layer.py -q -x -k "smid_gating or overlapping or device_split" >> $O/smid.log 2>&1; echo "smid rep $i rc=$?"
done
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
timeout 900 python bench.py > $O/bench_arxiv.json 2> $O/bench_arxiv.err; echo "bench3 rc=$?"
echo done
