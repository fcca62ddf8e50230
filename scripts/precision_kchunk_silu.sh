# R-4e follow-up: chunk only the gate_up GEMM (BULLET_GEMM_KCHUNK_ONLY=silu),
# layer error at Qwen2.5-14B / Llama-3.1-8B dims and the bench cost, both modes.
export BULLET_GEMM_KCHUNK_ONLY=${ONLY:-silu}
for mode in splitk onchip; do
  for dims in "5120 40 8 13824 57" "4096 32 8 14336 57"; do
    echo "== dims=$dims kc=${KC:-1024} mode=$mode only=$BULLET_GEMM_KCHUNK_ONLY"
    BULLET_GEMM_KCHUNK_MODE=$mode BULLET_GEMM_KCHUNK=${KC:-1024} timeout 400 python tests/tools/diag_layer.py $dims 2>&1 | grep "kind=4"
  done
  BULLET_GEMM_KCHUNK_MODE=$mode BULLET_GEMM_KCHUNK=${KC:-1024} timeout 600 python bench.py --no-cpu-baseline --p 76 --k 8 > gpurun_out/v7_${BULLET_GEMM_KCHUNK_ONLY}_$mode.log 2>>gpurun_out/v7.err
done
unset BULLET_GEMM_KCHUNK_ONLY
timeout 600 python bench.py --no-cpu-baseline --p 76 --k 8 > gpurun_out/v7_base.log 2>>gpurun_out/v7.err
