O=gpurun_out/r02; mkdir -p $O
timeout 1200 python scripts/fit_perfmodel.py $O/perf_params_b200.json > $O/l_fit.log 2>&1
cp $O/perf_params_b200.json $O/perf_params_b200_points.json profiles/ 2>/dev/null
timeout 900 python bench.py --sweep --no-cpu-baseline > $O/l_bench3.json 2> $O/l_bench3.err
timeout 900 python bench.py --config sharegpt-8b --sweep --no-cpu-baseline > $O/l_bench2.json 2> $O/l_bench2.err
timeout 900 python -m pytest tests -m gpu -q > $O/l_tests.log 2>&1
echo done
