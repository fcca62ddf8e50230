#!/bin/bash
set -u
mkdir -p gpurun_out/s1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s1/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/s1/tests.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/s1/tests.log
timeout 900 python bench.py > gpurun_out/s1/bench.json 2> gpurun_out/s1/bench.err; echo "bench rc=$?"
tail -c 600 gpurun_out/s1/bench.json
