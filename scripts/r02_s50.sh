OUT=s50 bash scripts/r02_s49.sh
mkdir -p gpurun_out/s50; timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_tp_peer.py -q -x -k "accumulation or gemm or peer" > gpurun_out/s50/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/s50/tests.log
