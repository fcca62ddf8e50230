# R-4e experiment: layer error vs oracle with every long-K GEMM accumulated in
# K chunks (BULLET_GEMM_KCHUNK=kc; BULLET_GEMM_KCHUNK_MODE=onchip (default) | splitk)
for dims in "5120 40 8 13824 57" "4096 32 8 14336 57" "8192 64 8 28672 57"; do
  for kc in ${KCS:-0 2048 1024 512}; do
    echo "== dims=$dims kc=$kc mode=${BULLET_GEMM_KCHUNK_MODE:-onchip}"
    BULLET_GEMM_KCHUNK=$kc BULLET_GEMM_DEBUG=1 timeout 400 python tests/tools/diag_layer.py $dims > /tmp/d.log 2>&1
    grep -v "^gemm" /tmp/d.log | tail -4
    grep "^gemm" /tmp/d.log | sort | uniq | head -5
  done
done
