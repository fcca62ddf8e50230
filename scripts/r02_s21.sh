#!/bin/bash
# Driver-path checks on the closing kernels: the reference (oracle) arm, and a 2-process TP bench on the
# 1-GPU lease (ranks share the GPU: gloo; numbers meaningless, the rank-agreed split is what is checked).
set -u
O=gpurun_out/s21; mkdir -p $O
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/ref.json 2> $O/ref.err; echo "ref rc=$?"; tail -c 400 $O/ref.json
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 3 --no-cpu-baseline > $O/tp2.json 2> $O/tp2.err; echo "tp2 rc=$?"; tail -c 600 $O/tp2.json
echo done
