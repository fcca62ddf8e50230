O=gpurun_out/r02; mkdir -p $O
timeout 1200 python scripts/fit_perfmodel.py $O/m_perf_params_b200.json > $O/m_fit.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -k "die_probe or long_context" -q > $O/m_tests.log 2>&1
timeout 600 python scripts/die_sigma.py --config sharegpt-8b --p 76 --k 8 > $O/m_die_sigma2.jsonl 2> $O/m_die_sigma2.err
timeout 600 python scripts/die_sigma.py --config arxiv-8b --p 84 --k 5 > $O/m_die_sigma3.jsonl 2> $O/m_die_sigma3.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --config qwen14b-tp2 --steps 3 --warmup 3 --k-max 4 > $O/m_tp2.json 2> $O/m_tp2.err
echo done
