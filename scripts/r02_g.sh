O=gpurun_out/r02; mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_layer.py -k "pool" -x -q > $O/g_pool.log 2>&1
timeout 300 python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1 > $O/g_trace_dec2.jsonl 2>&1
echo done
