O=gpurun_out/r02; mkdir -p $O
timeout 1500 python scripts/fit_perfmodel.py $O/o_perf_params_b200.json > $O/o_fit.log 2>&1
echo done
