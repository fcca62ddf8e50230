#!/bin/bash
# Refit the performance model on the closing kernels (new file; compared before adoption).
set -u
O=gpurun_out/refit; mkdir -p $O
timeout 2400 python scripts/fit_perfmodel.py $O/perf_params_b200_r02b.json > $O/fit.log 2>&1; echo "fit rc=$?"; tail -3 $O/fit.log
